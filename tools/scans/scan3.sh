L=paper_conf_cluster_chenwttm18_b200
rm -f gpurun_out/tl.txt
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl.txt SAT_LIBRARY=$L/libsat_tl.so python tools/shape_scan.py 0 16384x16384 9088x16384 8192x8192 4096x65536
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl.txt SAT_LIBRARY=$L/libsat_tl.so python tools/shape_scan.py 1 16384x16384
python tools/tl_analyze.py gpurun_out/tl.txt
