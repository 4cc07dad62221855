# Short/wide images: short-band variant and cluster size per pair.
for rep in 1 2; do
for cfg in "SAT_SHORT=0" "SAT_SHORT=1" "SAT_CLUSTER=1" "SAT_CLUSTER=8"; do echo "== $cfg";
  for p in 0 1 2; do env $cfg timeout 120 python tools/shape_scan.py $p 4096x65536 3072x65536; done; done
done
