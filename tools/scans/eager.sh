L=paper_conf_cluster_chenwttm18_b200
SAT_LIBRARY=$L/libsat_eager.so timeout 120 python -c "import __graft_entry__ as g; g.smoke()"
for rep in 1 2; do for v in libsat_ref libsat_eager; do
echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 1080x1920x256
SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 2 16384x16384
done; done
