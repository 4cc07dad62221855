L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat_ref libsat_land1k libsat_land1k4; do
echo "== $v"; SAT_LOG=1 SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x256 2>&1 | grep -v "epoch=[0-9]*[1-9]$" | grep "pair=\|grid" | head -8
SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
done; done
