L=paper_conf_cluster_chenwttm18_b200
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
python tools/shape_scan.py 0 16384x16384 8192x8192 9088x16384 1080x1920x1024 4096x65536
python tools/shape_scan.py 1 16384x16384 8192x8192 65536x4096
python tools/shape_scan.py 2 16384x16384 4096x65536
STEPS=1 SAT_LIBRARY=$L/libsat_prof.so python tools/shape_scan.py 0 16384x16384 9088x16384 2>&1 | grep -v "^pair" | tail -4
