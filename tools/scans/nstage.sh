L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do
for v in libsat libsat_n8_3 libsat_n8_6; do echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 120 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x1024; done
for v in libsat libsat_n32_2 libsat_n32_5; do echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 120 python tools/shape_scan.py 1 16384x16384 8192x8192 65536x4096; done
done
