"""Where do the bench's occasional slow steps come from?  (diagnostic, not a test)

1. host: a busy loop in 1 ms slices for 5 s; reports slices that took > 5 ms (the
   process was descheduled or the host stalled);
2. device only: 150 iterations of a ~30 ms chain of elementwise kernels, no host
   synchronisation, one event per iteration (GPU-side disturbance shows here);
3. device + host syncs: the same iterations split into 25 pieces with a
   synchronize after each (the library's round loop synchronises with the host).
"""
import json
import statistics
import time

import torch


def host_probe(seconds=5.0):
    slices = []
    t_end = time.perf_counter() + seconds
    while time.perf_counter() < t_end:
        t0 = time.perf_counter()
        while time.perf_counter() - t0 < 1e-3:
            pass
        slices.append((time.perf_counter() - t0) * 1e3)
    big = sorted(s for s in slices if s > 5.0)
    return {"slices": len(slices), "over_5ms": len(big), "worst_ms": big[-5:]}


def dev_probe(sync_pieces):
    x = torch.empty(1 << 26, device="cuda")  # 256 MB: one pass ~0.08 ms
    x.fill_(1.0)

    def piece(n):
        for _ in range(n):
            x.mul_(1.0000001)

    per_iter = 360  # ~30 ms
    for _ in range(5):
        piece(per_iter)
    torch.cuda.synchronize()
    evs = [torch.cuda.Event(enable_timing=True) for _ in range(151)]
    evs[0].record()
    for i in range(150):
        if sync_pieces:
            for _ in range(sync_pieces):
                piece(per_iter // sync_pieces)
                torch.cuda.synchronize()
        else:
            piece(per_iter)
        evs[i + 1].record()
    torch.cuda.synchronize()
    ms = [evs[i].elapsed_time(evs[i + 1]) for i in range(150)]
    med = statistics.median(ms)
    return {"median_ms": round(med, 3), "max_ms": round(max(ms), 3),
            "over_1.25x": sum(m > 1.25 * med for m in ms), "worst": sorted(round(m, 2) for m in ms)[-5:]}


if __name__ == "__main__":
    out = {"host": host_probe(), "device_only": dev_probe(0), "device_synced": dev_probe(25),
           "host_again": host_probe()}
    print(json.dumps(out))
