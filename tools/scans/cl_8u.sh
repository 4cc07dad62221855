# Cluster size for the byte-input pairs at 224-512 bands.
for rep in 1 2; do
for cl in 4 8; do echo "== SAT_CLUSTER=$cl"; SAT_CLUSTER=$cl timeout 120 python tools/shape_scan.py 0 7168x8192 8192x8192 12288x8192 16384x16384; done
done
