L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat libsat_nolb libsat_x1 libsat_x2 libsat_x3; do
echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 9088x16384
done; done
