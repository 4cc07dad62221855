# round profile set: ncu --set full of the top kernel per workload + the bench launch list
O=gpurun_out/prof
mkdir -p $O
timeout 300 python tools/context_bench.py 10 > $O/context.json 2> $O/context.err
for cfg in "0 16384 16384 1 p0_16384x16384x1" "0 8192 8192 1 p0_8192x8192x1" "0 1080 1920 1024 p0_1080x1920x1024" "1 16384 16384 1 p1_16384x16384x1" "1 65536 65536 1 p1_65536x65536x1" "2 16384 16384 1 p2_16384x16384x1" "3 16384 16384 1 p3_16384x16384x1" "4 16384 16384 1 p4_16384x16384x1"; do
  set -- $cfg
  timeout 240 ncu --set full --clock-control none --import-source on -k regex:sat_tile -s 2 -c 1 -f -o $O/$5 python tools/prof_one.py $1 $2 $3 $4 3 > $O/$5.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_bench.csv python bench.py --steps 20 --warmup 5 > $O/bench_under_ncu.log 2>&1
ls -la $O
