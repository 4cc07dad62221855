L=paper_conf_cluster_chenwttm18_b200
for cl in 1 4; do echo "== nolbprof CL=$cl"; STEPS=2 SAT_CLUSTER=$cl SAT_LIBRARY=$L/libsat_nolbprof.so timeout 60 python tools/shape_scan.py 0 16384x16384 9088x16384 2>&1 | tail -4; done
echo "== prof real CL=4"; STEPS=2 SAT_LIBRARY=$L/libsat_prof.so timeout 60 python tools/shape_scan.py 0 9088x16384 2>&1 | tail -2
