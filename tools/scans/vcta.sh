L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat_ref libsat_vcta; do
echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x256
SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
done; done
