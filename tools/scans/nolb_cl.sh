L=paper_conf_cluster_chenwttm18_b200
for cl in 1 4 8; do echo "== nolb CL=$cl"; SAT_CLUSTER=$cl SAT_LIBRARY=$L/libsat_nolb.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 9088x16384; done
for cl in 1 4 8; do echo "== real CL=$cl"; SAT_CLUSTER=$cl timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 9088x16384; done
