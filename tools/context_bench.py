"""Same-box context for the SAT numbers (development
tool, not the bench contract): the libraries the paper compares against
(Table II), run on this B200.

  * NPP nppiIntegral_8u32s_C1R / nppiIntegral_8u32f_C1R (CUDA 12.9 NPP): the
    exclusive (H+1) x (W+1) integral of PAPER.md:63-68 / Eq. 2.
  * torch: x.cumsum(0).cumsum(1) in the output dtype (two passes; the plain
    library composition of the definition).
  * libsat sat_compute (this repo), same inputs.

All timed with CUDA events on the default stream (NPP's non-Ctx entry points
use it), L2 flushed between steps when the working set is below 4x L2.
Prints one JSON object; python tools/context_bench.py [STEPS]
"""
import ctypes
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen


class NppiSize(ctypes.Structure):
    _fields_ = [("width", ctypes.c_int), ("height", ctypes.c_int)]


def npp():
    for name in ("libnppist.so.12", "libnppist.so", "/usr/local/cuda/lib64/libnppist.so"):
        try:
            return ctypes.CDLL(name)
        except OSError:
            pass
    return None


L2 = 126 << 20
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timeit(fn, steps, bytes_ws):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(steps):
        if bytes_ws < 4 * L2:
            flush.add_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
    lib = npp()
    res = {"device": torch.cuda.get_device_name(), "steps": steps, "entries": []}
    for (H, W) in [(4096, 4096), (8192, 8192), (16384, 16384)]:
        px = H * W
        x = torch.empty((H, W), dtype=torch.uint8, device="cuda")
        satgen.fill_device(x, seed=1001)
        ws = px * 5
        ours_out = torch.empty((H, W), dtype=torch.int32, device="cuda")
        ms = timeit(lambda: sat.sat(x, out=ours_out), steps, ws)
        res["entries"].append({"impl": "libsat sat_compute", "pair": "8u->32s", "shape": f"{H}x{W}",
                               "ms": ms, "gpx_s": px / ms / 1e6, "alg_gbs": ws / ms / 1e6})
        # SAT consumers (N4): box sums of radius 8 from the SAT (reads S, writes out: 8 B/px)
        bo = torch.empty((H, W), dtype=torch.int32, device="cuda")
        ms = timeit(lambda: sat.box_filter(ours_out, 8, 8, out=bo), steps, px * 8)
        res["entries"].append({"impl": "libsat sat_box_filter r=8 (from SAT)", "pair": "32s->32s",
                               "shape": f"{H}x{W}", "ms": ms, "gpx_s": px / ms / 1e6,
                               "alg_gbs": px * 8 / ms / 1e6})
        del bo
        nq = 1 << 22
        rq = torch.randint(0, min(H, W), (nq, 4), dtype=torch.int32, device="cuda")
        ms = timeit(lambda: sat.rect_sums(ours_out, rq), steps, nq * 20)
        res["entries"].append({"impl": "libsat sat_rect_sums 4M random rects", "pair": "32s",
                               "shape": f"{H}x{W}", "ms": ms, "gqueries_s": nq / ms / 1e6})
        del rq
        # NPP-style pitched output (rows padded to 16 B, like nppiMalloc)
        ex_out = torch.empty((H + 1, W + 4), dtype=torch.int32, device="cuda")[:, :W + 1]
        ms = timeit(lambda: sat.sat_exclusive(x, full=True, out=ex_out), steps, ws)
        res["entries"].append({"impl": "libsat sat_compute_exclusive (H+1)x(W+1)", "pair": "8u->32s",
                               "shape": f"{H}x{W}", "ms": ms, "gpx_s": px / ms / 1e6,
                               "alg_gbs": ws / ms / 1e6})
        ex_f = torch.empty((H + 1, W + 4), dtype=torch.float32, device="cuda")[:, :W + 1]
        ms = timeit(lambda: sat.sat_exclusive(x, full=True, out=ex_f), steps, ws)
        res["entries"].append({"impl": "libsat sat_compute_exclusive 8u->32f (H+1)x(W+1)",
                               "pair": "8u->32f", "shape": f"{H}x{W}", "ms": ms,
                               "gpx_s": px / ms / 1e6, "alg_gbs": ws / ms / 1e6})
        del ex_f
        if lib is not None:
            for name, dt, fn in (("nppiIntegral_8u32s_C1R", torch.int32, lib.nppiIntegral_8u32s_C1R),
                                 ("nppiIntegral_8u32f_C1R", torch.float32, lib.nppiIntegral_8u32f_C1R)):
                o = torch.empty((H + 1, W + 1), dtype=dt, device="cuda")
                if dt == torch.int32:
                    fn.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                   NppiSize, ctypes.c_int32]
                    nval = ctypes.c_int32(0)
                else:
                    fn.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
                                   NppiSize, ctypes.c_float]
                    nval = ctypes.c_float(0.0)
                st = fn(x.data_ptr(), W, o.data_ptr(), (W + 1) * 4, NppiSize(W, H), nval)
                torch.cuda.synchronize()
                entry = {"impl": name, "pair": "8u->" + ("32s" if dt == torch.int32 else "32f"),
                         "shape": f"{H}x{W}", "status": int(st)}
                if st == 0:
                    # agreement with libsat on the interior (exclusive layout shifted by one)
                    if dt == torch.int32:
                        entry["matches_libsat"] = bool(torch.equal(o[1:, 1:], ours_out))
                        entry["matches_libsat_exclusive"] = bool(torch.equal(o, ex_out))
                    ms = timeit(lambda: fn(x.data_ptr(), W, o.data_ptr(), (W + 1) * 4, NppiSize(W, H), nval),
                                steps, ws)
                    entry.update({"ms": ms, "gpx_s": px / ms / 1e6, "alg_gbs": ws / ms / 1e6})
                res["entries"].append(entry)
                del o
        for name, dt in (("torch cumsum(0).cumsum(1) int32", torch.int32),):
            o = torch.empty((H, W), dtype=dt, device="cuda")

            def f():
                torch.cumsum(x, 0, dtype=dt, out=o)
                torch.cumsum(o, 1, out=o)

            ms = timeit(f, steps, ws)
            res["entries"].append({"impl": name, "pair": "8u->32s", "shape": f"{H}x{W}", "ms": ms,
                                   "gpx_s": px / ms / 1e6, "alg_gbs": ws / ms / 1e6})
            del o
        xf = torch.empty((H, W), dtype=torch.float32, device="cuda")
        satgen.fill_device(xf, seed=1001)
        of = torch.empty((H, W), dtype=torch.float32, device="cuda")
        ms = timeit(lambda: sat.sat(xf, out=of), steps, px * 8)
        res["entries"].append({"impl": "libsat sat_compute", "pair": "32f->32f", "shape": f"{H}x{W}",
                               "ms": ms, "gpx_s": px / ms / 1e6, "alg_gbs": px * 8 / ms / 1e6})

        def g():
            torch.cumsum(xf, 0, out=of)
            torch.cumsum(of, 1, out=of)

        ms = timeit(g, steps, px * 8)
        res["entries"].append({"impl": "torch cumsum(0).cumsum(1) float32", "pair": "32f->32f",
                               "shape": f"{H}x{W}", "ms": ms, "gpx_s": px / ms / 1e6,
                               "alg_gbs": px * 8 / ms / 1e6})
        del x, xf, of, ours_out, ex_out
        torch.cuda.empty_cache()
    print(json.dumps(res))


if __name__ == "__main__":
    main()
