L=paper_conf_cluster_chenwttm18_b200
SAT_SHORT=1 timeout 400 python -m pytest tests/test_parity_gpu.py -x -q -k "shapes or padded or batched_with or full_size_sampled or band_with or in_place or wraps" > gpurun_out/short_tests.log 2>&1; echo rc=$? >> gpurun_out/short_tests.log
for rep in 1 2; do for sh in 0 1; do
echo "== short=$sh"; SAT_SHORT=$sh timeout 60 python tools/shape_scan.py 0 4096x65536 2048x65536 8192x8192 4096x4096 1080x1920x4
SAT_SHORT=$sh timeout 60 python tools/shape_scan.py 1 4096x65536 8192x8192
SAT_SHORT=$sh timeout 60 python tools/shape_scan.py 2 4096x65536 16384x16384
done; done
echo "== default"; timeout 60 python tools/shape_scan.py 0 4096x65536 16384x16384 8192x8192; timeout 60 python tools/shape_scan.py 2 4096x65536 65536x4096
