# wait-policy A/B (same box): suspend-hint try_wait vs test_wait + nanosleep polling
L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat_s0 libsat_lb128 libsat_b64 libsat_b128 libsat_p128 libsat_lb64b32 libsat_all; do
echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x256
SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
done; done
