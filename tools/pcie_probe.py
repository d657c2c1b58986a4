"""Host<->device copy ceilings on the box (pinned buffers): one large copy per
direction, both directions at once, and 36 copies of the C2 batch sizes.
Developer tool (sets the e2e roof)."""
import time

import torch


def main():
    torch.cuda.set_device(0)
    MB = 1 << 20
    for size in (24 * MB, 248 * MB):
        h = torch.empty(size, dtype=torch.uint8).pin_memory()
        d = torch.empty(size, dtype=torch.uint8, device="cuda")
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        for _ in range(2):
            d.copy_(h, non_blocking=True)
            h.copy_(d, non_blocking=True)
        torch.cuda.synchronize()
        t = time.perf_counter(); d.copy_(h, non_blocking=True); torch.cuda.synchronize(); th = time.perf_counter() - t
        t = time.perf_counter(); h.copy_(d, non_blocking=True); torch.cuda.synchronize(); td = time.perf_counter() - t
        h2 = torch.empty(size, dtype=torch.uint8).pin_memory()
        d2 = torch.empty(size, dtype=torch.uint8, device="cuda")
        torch.cuda.synchronize()
        t = time.perf_counter()
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.synchronize()
        tb = time.perf_counter() - t
        print(f"{size / MB:5.0f} MB: H2D {size / th / 1e9:6.1f} GB/s  D2H {size / td / 1e9:6.1f} GB/s  "
              f"both at once {2 * size / tb / 1e9:6.1f} GB/s total", flush=True)
    # 36 copies of 0.25 / 1 MB (the C2 batch)
    hs = [torch.empty(sz, dtype=torch.uint8).pin_memory() for sz in [MB, MB // 4] * 18]
    ds = [torch.empty(h.numel(), dtype=torch.uint8, device="cuda") for h in hs]
    for _ in range(2):
        for h, d in zip(hs, ds):
            d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    t = time.perf_counter()
    for h, d in zip(hs, ds):
        d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    tt = time.perf_counter() - t
    tot = sum(h.numel() for h in hs)
    print(f"36 H2D copies ({tot / MB:.1f} MB): {tot / tt / 1e9:6.1f} GB/s, {tt * 1e6 / 36:.1f} us per copy")


if __name__ == "__main__":
    main()
