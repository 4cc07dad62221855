L=paper_conf_cluster_chenwttm18_b200
SAT_LIBRARY=$L/libsat_t64.so timeout 120 python -c "import __graft_entry__ as g; g.smoke()"
for rep in 1 2; do for v in libsat libsat_t64; do
echo "== $v"; SAT_LOG=1 SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536 9088x16384 1080x1920x256 2>&1 | grep -v "^\[libsat\]" 
for cl in 8; do SAT_CLUSTER=$cl SAT_LIBRARY=$L/$v.so timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 | sed "s/^/CL$cl /"; done
done; done
SAT_LOG=1 SAT_LIBRARY=$L/libsat_t64.so timeout 60 python tools/shape_scan.py 0 16384x16384 2>&1 | grep "libsat\]" | head -2
