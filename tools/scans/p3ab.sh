L=paper_conf_cluster_chenwttm18_b200
for rep in 1 2; do for v in libsat libsat_narrow; do echo "== $v"; SAT_LIBRARY=$L/$v.so timeout 60 python - <<'PY'
import sys, torch, statistics
sys.path.insert(0, '.')
import paper_conf_cluster_chenwttm18_b200 as sat, satgen
for H, W in ((16384, 16384), (8192, 8192), (65536, 4096), (4096, 65536)):
    x = torch.empty((H, W), dtype=torch.uint8, device="cuda"); satgen.fill_device(x, seed=1)
    y = torch.empty((H, W), dtype=torch.float32, device="cuda")
    for _ in range(3): sat.sat(x, out=y)
    torch.cuda.synchronize(); ts = []
    for _ in range(10):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); sat.sat(x, out=y); b.record(); torch.cuda.synchronize(); ts.append(a.elapsed_time(b))
    ms = statistics.median(ts); print(H, W, round(ms, 4), round(H * W * 5 / ms / 1e6 / 6545.9, 3))
PY
done; done
