O=gpurun_out/prof
mkdir -p $O
for cfg in "1 65536 65536 1 p1_65536x65536x1" "2 16384 16384 1 p2_16384x16384x1" "3 16384 16384 1 p3_16384x16384x1" "4 16384 16384 1 p4_16384x16384x1"; do
  set -- $cfg
  timeout 240 ncu --set full --clock-control none --import-source on -k regex:sat_tile -s 2 -c 1 -f -o $O/$5 python tools/prof_one.py $1 $2 $3 $4 3 > $O/$5.log 2>&1
done
ls -la $O
