L=paper_conf_cluster_chenwttm18_b200
rm -f gpurun_out/tlnl*.txt
STEPS=1 SAT_CLUSTER=1 SAT_TIMELINE_OUT=gpurun_out/tlnl1.txt SAT_LIBRARY=$L/libsat_nolbtl.so python tools/shape_scan.py 0 9088x16384
python tools/tl_analyze.py gpurun_out/tlnl1.txt
STEPS=1 SAT_CLUSTER=4 SAT_TIMELINE_OUT=gpurun_out/tlnl4.txt SAT_LIBRARY=$L/libsat_nolbtl.so python tools/shape_scan.py 0 9088x16384
python tools/tl_analyze.py gpurun_out/tlnl4.txt
