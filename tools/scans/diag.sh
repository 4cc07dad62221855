L=paper_conf_cluster_chenwttm18_b200
for v in libsat libsat_nolb libsat_prof; do echo "== $v"; SAT_LIBRARY=$L/$v.so python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 2>&1 | grep -v Warn; done
echo "== 32f nolb"; SAT_LIBRARY=$L/libsat_nolb.so python tools/shape_scan.py 1 16384x16384 8192x8192
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl_16k.txt SAT_LIBRARY=$L/libsat_tl.so python tools/shape_scan.py 0 16384x16384
python tools/tl_analyze.py gpurun_out/tl_16k.txt
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl_8k.txt SAT_LIBRARY=$L/libsat_tl.so python tools/shape_scan.py 0 8192x8192
python tools/tl_analyze.py gpurun_out/tl_8k.txt
