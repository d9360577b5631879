"""Pinned D2H / H2D bandwidth of 746 MB (one bench step's 4K output), with the process bound to all cores vs to the
GPU-local NUMA node's cores (pinned pages first-touched there)."""
import os
import sys
import time

import torch


def bw(label):
    n = 746_496_000
    d = torch.empty(n, dtype=torch.uint8, device="cuda")
    h = torch.empty(n, dtype=torch.uint8).pin_memory()
    for _ in range(2):
        h.copy_(d, non_blocking=True)
        d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
    e0.record()
    for _ in range(5):
        h.copy_(d, non_blocking=True)
    e1.record()
    for _ in range(5):
        d.copy_(h, non_blocking=True)
    e2.record()
    torch.cuda.synchronize()
    print(f"{label}: D2H {5 * n / e0.elapsed_time(e1) / 1e6:.1f} GB/s  H2D {5 * n / e1.elapsed_time(e2) / 1e6:.1f} GB/s",
          flush=True)


p = torch.cuda.get_device_properties(0)
bus = getattr(p, "pci_bus_id", None)
print("props:", {k: getattr(p, k, None) for k in ("pci_bus_id", "pci_device_id", "pci_domain_id")})
bw("all cores")
if bus is not None:
    path = f"/sys/bus/pci/devices/{getattr(p, 'pci_domain_id', 0):04x}:{bus:02x}:{getattr(p, 'pci_device_id', 0):02x}.0"
    try:
        node = open(path + "/numa_node").read().strip()
        cpus = open(path + "/local_cpulist").read().strip()
        print("numa node", node, "local cpus", cpus)
        sel = set()
        for part in cpus.split(","):
            a, _, b = part.partition("-")
            sel |= set(range(int(a), int(b or a) + 1))
        os.sched_setaffinity(0, sel & os.sched_getaffinity(0) or os.sched_getaffinity(0))
        bw("GPU-local cores")
    except OSError as exc:
        print("no sysfs numa info:", exc)
