"""PCIe probe for the e2e leg: pinned H2D / D2H bandwidth alone and concurrent
(the ceiling of spaden_spmv_host_batched).  Prints one JSON line."""
import json

import torch


def main(nbytes=4 * 1497600, reps=44):
    dev = torch.device("cuda:0")
    h = [torch.empty(nbytes // 4, dtype=torch.float32).pin_memory() for _ in range(2)]
    d = [torch.empty(nbytes // 4, dtype=torch.float32, device=dev) for _ in range(2)]
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)

    def timed(fn):
        fn()
        torch.cuda.synchronize(dev)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        s1.wait_event(e0)
        s2.wait_event(e0)
        fn()
        a, b = torch.cuda.Event(), torch.cuda.Event()
        a.record(s1)
        b.record(s2)
        torch.cuda.current_stream().wait_event(a)
        torch.cuda.current_stream().wait_event(b)
        e1.record()
        torch.cuda.synchronize(dev)
        return e0.elapsed_time(e1) / reps

    def h2d():
        with torch.cuda.stream(s1):
            for _ in range(reps):
                d[0].copy_(h[0], non_blocking=True)

    def d2h():
        with torch.cuda.stream(s2):
            for _ in range(reps):
                h[1].copy_(d[1], non_blocking=True)

    def both():
        h2d()
        d2h()

    out = {}
    for it in range(3):
        for name, fn in (("h2d", h2d), ("d2h", d2h), ("both", both)):
            ms = timed(fn)
            out[f"{name}_{it}"] = {"ms_per_copy": ms, "GBps_per_direction": nbytes / (ms * 1e-3) / 1e9}
    out["bytes"] = nbytes
    print(json.dumps(out))


if __name__ == "__main__":
    main()
