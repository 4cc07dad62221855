L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for cl in 4 8 16; do
echo "== CL=$cl"; SAT_CLUSTER=$cl SAT_LOG=1 SAT_LIBRARY=$L/libsat_cl16.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 2>&1 | grep -v "epoch=[0-9]*[02-9]$" | grep "pair=\|grid" | cut -c1-150
SAT_CLUSTER=$cl SAT_LIBRARY=$L/libsat_cl16.so timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
done; done
