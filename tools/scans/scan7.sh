L=paper_conf_cluster_chenwttm18_b200
rm -f gpurun_out/tl7.txt gpurun_out/tl7b.txt
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl7.txt SAT_LIBRARY=$L/libsat_tlnolb.so python tools/shape_scan.py 0 9088x16384
STEPS=1 SAT_CLUSTER=1 SAT_TIMELINE_OUT=gpurun_out/tl7b.txt SAT_LIBRARY=$L/libsat_tl.so python tools/shape_scan.py 0 9088x16384
python tools/tl_analyze.py gpurun_out/tl7.txt
python tools/tl_analyze.py gpurun_out/tl7b.txt
