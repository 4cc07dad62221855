S="1024x16384 2048x16384 4096x16384 8192x16384 9088x16384 12288x16384 16384x16384 18176x16384 24576x16384 32768x16384 16384x8192 16384x32768 8192x8192"
echo "== main"; python tools/shape_scan.py 0 $S
echo "== nolb"; SAT_LIBRARY=paper_conf_cluster_chenwttm18_b200/libsat_nolb.so python tools/shape_scan.py 0 $S
echo "== CL1"; SAT_CLUSTER=1 python tools/shape_scan.py 0 16384x16384 8192x8192
echo "== CL8"; SAT_CLUSTER=8 python tools/shape_scan.py 0 16384x16384 8192x8192
echo "== prof"; STEPS=2 SAT_LIBRARY=paper_conf_cluster_chenwttm18_b200/libsat_prof.so python tools/shape_scan.py 0 16384x16384 8192x8192 9088x16384 2>&1 | grep -v "^pair"
