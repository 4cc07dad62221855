# Cluster size for the float pairs around the 264-band threshold.
for rep in 1 2; do
for cl in 0 4 8; do echo "== SAT_CLUSTER=$cl"; SAT_CLUSTER=$cl timeout 120 python tools/shape_scan.py 1 8192x8192 8448x8192 6144x16384 4096x4096; SAT_CLUSTER=$cl timeout 120 python tools/shape_scan.py 2 8192x8192 4096x8192; done
done
