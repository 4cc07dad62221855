O=gpurun_out/prof
mkdir -p $O
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench.csv python bench.py --steps 20 --warmup 5 > $O/bench_under_ncu.log 2>&1
for cfg in "0 16384 16384 1 p0_16384x16384x1" "0 8192 8192 1 p0_8192x8192x1" "0 1080 1920 1024 p0_1080x1920x1024" "1 16384 16384 1 p1_16384x16384x1"; do
  set -- $cfg
  timeout 240 ncu --set full --clock-control none --import-source on -k regex:sat_tile -s 2 -c 1 -f -o $O/$5 python tools/prof_one.py $1 $2 $3 $4 3 > $O/$5.log 2>&1
done
ls -la $O
