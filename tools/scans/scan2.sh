S="16384x16384 8192x8192 9088x16384 1080x1920x1024 4096x65536"
L=paper_conf_cluster_chenwttm18_b200
for v in libsat libsat_th16 libsat_th16l5 libsat_th8; do for cl in 4 8; do
echo "== $v CL=$cl"; SAT_CLUSTER=$cl SAT_LIBRARY=$L/$v.so python tools/shape_scan.py 0 $S
done; done
