L=paper_conf_cluster_chenwttm18_b200
rm -f gpurun_out/tl8*.txt
for v in tl tl_l7 tl_l2; do
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl8_$v.txt SAT_LIBRARY=$L/libsat_$v.so python tools/shape_scan.py 1 8448x16384
python tools/tl_analyze.py gpurun_out/tl8_$v.txt | awk 'NR<=3 || NR%4==0'
done
STEPS=1 SAT_TIMELINE_OUT=gpurun_out/tl8_8u_l2.txt SAT_LIBRARY=$L/libsat_tl_l2.so python tools/shape_scan.py 0 9088x16384
python tools/tl_analyze.py gpurun_out/tl8_8u_l2.txt | awk 'NR<=3 || NR%4==0'
bash tools/scans/ab.sh "16384x16384 8192x8192 8448x16384 65536x4096" 1 libsat libsat_l7
