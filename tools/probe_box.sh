#!/bin/bash
# One-shot probe of the GPU box's host side (cores, memory, tmpfs, PCIe link) for DESIGN.md.
out=gpurun_out/probe_box.txt
{
echo "== nproc"; nproc; python -c 'import os;print("affinity",len(os.sched_getaffinity(0)))'
echo "== lscpu"; lscpu | head -30
echo "== numa"; lscpu | grep -i numa; cat /sys/fs/cgroup/cpu.max 2>/dev/null
echo "== mem"; free -g; df -h /dev/shm /tmp
echo "== gpu"; nvidia-smi -L; nvidia-smi --query-gpu=index,pci.bus_id,pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,clocks.sm,clocks.max.sm --format=csv
nvidia-smi topo -m
for d in /sys/bus/pci/devices/*; do if [ -f $d/numa_node ] && grep -q 0x10de $d/vendor 2>/dev/null; then echo "$d numa=$(cat $d/numa_node) class=$(cat $d/class)"; fi; done
echo "== kernel"; uname -a; cat /proc/sys/kernel/perf_event_paranoid
echo "== h2d"
python - <<'PY'
import torch, time
torch.cuda.init()
p = torch.cuda.get_device_properties(0); print(p)
for sz in [1<<18, 1<<20, 16<<20, 256<<20, 1<<30]:
    h = torch.empty(sz, dtype=torch.uint8).pin_memory(); d = torch.empty(sz, dtype=torch.uint8, device='cuda')
    for _ in range(3): d.copy_(h, non_blocking=True)
    torch.cuda.synchronize()
    n = max(4, (4<<30)//sz)
    s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(n): d.copy_(h, non_blocking=True)
    e.record(); torch.cuda.synchronize()
    t = s.elapsed_time(e)/1e3
    print(f"H2D pinned {sz>>10} KiB x{n}: {sz*n/t/1e9:.1f} GB/s")
    s.record()
    for _ in range(n): h.copy_(d, non_blocking=True)
    e.record(); torch.cuda.synchronize()
    t = s.elapsed_time(e)/1e3
    print(f"D2H pinned {sz>>10} KiB x{n}: {sz*n/t/1e9:.1f} GB/s")
PY
} > $out 2>&1
cat $out
