"""Where the host-path (P:325 memcpy variant) time goes: plain pinned H2D/D2H
rates vs the ecl_mst call.   python tools/e2e_probe.py [--config road]"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_sc_fallingsb23_b200 as eclmst  # noqa: E402
import synth  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="road")
    ap.add_argument("--reps", type=int, default=7)
    a = ap.parse_args()
    g = synth.make_config(a.config, "full")
    h = [t.pin_memory() for t in (g.nindex, g.nlist, g.eweight)]
    out = torch.empty(g.M, dtype=torch.uint8).pin_memory()
    d = [torch.empty_like(t, device="cuda") for t in h]
    dm = torch.empty(g.M, dtype=torch.uint8, device="cuda")
    nbytes = sum(t.numel() * t.element_size() for t in h)

    def tm(fn):
        ts = []
        for _ in range(a.reps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            ts.append(time.perf_counter() - t0)
        ts.sort()
        return 1e3 * ts[len(ts) // 2]

    h2d = tm(lambda: [x.copy_(y, non_blocking=True) for x, y in zip(d, h)])
    d2h = tm(lambda: out.copy_(dm, non_blocking=True))
    e2e = tm(lambda: eclmst.ecl_mst(g.n, *h, out))
    ws = torch.empty(eclmst.ecl_mst_workspace_bytes(g.n, g.M), dtype=torch.uint8, device="cuda")
    dev = tm(lambda: eclmst.ecl_mst_device(g.n, *d, in_mst_out=dm, workspace=ws))
    print(f"{g.name}: H2D {nbytes / 1e6:.0f} MB {h2d:.2f} ms ({nbytes / h2d / 1e6:.1f} GB/s); "
          f"D2H {g.M / 1e6:.0f} MB {d2h:.2f} ms ({g.M / d2h / 1e6:.1f} GB/s); device run {dev:.2f} ms; "
          f"serial sum {h2d + d2h + dev:.2f} ms; ecl_mst e2e {e2e:.2f} ms")


if __name__ == "__main__":
    main()
