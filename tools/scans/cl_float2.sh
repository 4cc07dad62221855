# Cluster size for the float pairs between 192 and 256 bands.
for rep in 1 2; do
for cl in 4 8; do echo "== SAT_CLUSTER=$cl"; SAT_CLUSTER=$cl timeout 120 python tools/shape_scan.py 1 7168x8192 7680x8192 8192x8192 3584x32768; SAT_CLUSTER=$cl timeout 120 python tools/shape_scan.py 2 7168x8192 8192x8192; done
done
