# pacing scan: SAT_PACE_X / SAT_PACE_Y over the 8u and 32f headline shapes
for xy in "0 2" "8 1" "8 2" "16 1" "16 2" "32 2" "32 4" "4 2"; do
set -- $xy
echo "== X=$1 Y=$2"
SAT_PACE_X=$1 SAT_PACE_Y=$2 timeout 60 python tools/shape_scan.py 0 16384x16384 8192x8192 4096x65536
SAT_PACE_X=$1 SAT_PACE_Y=$2 timeout 60 python tools/shape_scan.py 1 16384x16384 8192x8192
done
