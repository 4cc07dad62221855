# 8u lookahead experiment (half-TMEM timing builds give wrong results; timing only)
L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat libsat_h3 libsat_h5 libsat_h7; do
echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x256
done; done
