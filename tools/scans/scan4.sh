L=paper_conf_cluster_chenwttm18_b200
STEPS=1 SAT_LIBRARY=$L/libsat_prof.so python tools/shape_scan.py 0 16384x16384 9088x16384 2>&1 | grep -v "^pair" | tail -4
STEPS=1 SAT_LIBRARY=$L/libsat_prof.so python tools/shape_scan.py 1 16384x16384 2>&1 | grep -v "^pair" | tail -2
