# Persistent-grid size vs wave quantisation (16384^2 8u: 128 cluster tickets of 4 bands).
for rep in 1 2; do
for fc in 0 64 66 70 72 74; do echo "== FORCE_CLUSTERS=$fc"; SAT_FORCE_CLUSTERS=$fc timeout 120 python tools/shape_scan.py 0 16384x16384 12288x16384; done
done
