#!/bin/bash
# One-off box survey: host/GPU facts + host-link bandwidth.
out=gpurun_out/box_facts.txt
{
echo "== nproc"; nproc
echo "== lscpu"; lscpu | head -20
echo "== free -g"; free -g
echo "== numactl"; (numactl -H 2>/dev/null || echo none)
echo "== nvidia-smi"; nvidia-smi
echo "== topo"; nvidia-smi topo -m
echo "== pcie"; nvidia-smi -q | grep -A12 -i 'PCI$\|GPU Link Info' | head -40
echo "== df"; df -h /tmp /root | head
} > $out 2>&1
python - >> $out 2>&1 <<'PY'
import torch, time
p = torch.cuda.get_device_properties(0)
print("props", p.name, p.multi_processor_count, "L2", getattr(p, "L2_cache_size", None), "mem", p.total_memory)
n = 1 << 30
h = torch.empty(n, dtype=torch.uint8).pin_memory()
d = torch.empty(n, dtype=torch.uint8, device="cuda")
for name, f in [("h2d", lambda: d.copy_(h, non_blocking=True)), ("d2h", lambda: h.copy_(d, non_blocking=True))]:
    best = 1e9
    for _ in range(10):
        s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); f(); e.record(); torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e))
    print(name, "GB/s", n / best / 1e6)
x = torch.empty(1 << 30, dtype=torch.int32, device="cuda").fill_(1)
best = 1e9
for _ in range(10):
    s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record(); y = x.sum(); e.record(); torch.cuda.synchronize(); best = min(best, s.elapsed_time(e))
print("read-only sum GB/s", 4 * (1 << 30) / best / 1e6)
PY
echo done >> $out
