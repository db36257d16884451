"""Pinned host->device copy ceiling on this box (the bound of bench.py's `e2e`).

Times, with CUDA events, (a) one copy of the default workload's H2D bytes as a
single pinned buffer and (b) the same bytes as the per-column copies the Q5
SF 1 e2e step issues (one cudaMemcpyAsync per column, same sizes).
"""
import json
import sys

import torch


def main():
    total = int(sys.argv[1]) if len(sys.argv) > 1 else 163324208
    dev = torch.device("cuda:0")
    s = torch.cuda.Stream()
    h = torch.empty(total, dtype=torch.uint8).pin_memory()
    d = torch.empty(total, dtype=torch.uint8, device=dev)
    # Q5 SF 1 column mix: 6 lineitem 4-/8-byte columns dominate (see bench.py e2e)
    n_li = 6001842
    sizes = [n_li * 4] * 6
    rest = total - sum(sizes)
    sizes += [rest // 10] * 9 + [rest - 9 * (rest // 10)]
    out = {}
    with torch.cuda.stream(s):
        for name, parts in (("single", [total]), ("per_column", sizes)):
            ms = []
            for it in range(8):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                off = 0
                for p in parts:
                    d[off:off + p].copy_(h[off:off + p], non_blocking=True)
                    off += p
                e1.record(s)
                e1.synchronize()
                if it >= 2:
                    ms.append(e0.elapsed_time(e1))
            best = min(ms)
            out[name] = {"bytes": total, "ms": best, "gbs": total / best / 1e6, "copies": len(parts)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
