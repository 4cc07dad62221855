# ncu --set full of the float 8192^2 configs after the cluster-size change (CL 8 from 224 bands).
O=gpurun_out/prof
mkdir -p $O
for cfg in "1 8192 8192 1 p1_8192x8192x1" "2 8192 8192 1 p2_8192x8192x1"; do
  set -- $cfg
  timeout 240 ncu --set full --clock-control none --import-source on -k regex:sat_tile -s 2 -c 1 -f -o $O/$5 python tools/prof_one.py $1 $2 $3 $4 3 > $O/$5.log 2>&1
done
ls -la $O
