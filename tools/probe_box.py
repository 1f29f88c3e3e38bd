"""Step-0 box probe: host link H2D/D2H/duplex size curve, HBM copy,
host facts. Writes gpurun_out/probe.json. Plumbing-only torch (pinned tensors, streams)."""
import json, os, subprocess, time, sys
import torch

def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:
        return f"ERR {e}"

out = {}
out["nvidia_smi_L"] = sh("nvidia-smi -L")
out["pcie"] = sh("nvidia-smi --query-gpu=index,pcie.link.gen.current,pcie.link.gen.max,pcie.link.width.current,pcie.link.width.max,memory.total --format=csv")
out["topo"] = sh("nvidia-smi topo -m")
out["lscpu"] = sh("lscpu")
out["free"] = sh("free -g")
out["numactl"] = sh("numactl -H 2>&1 || cat /sys/devices/system/node/node*/meminfo | head -20")
out["ulimit_l"] = sh("ulimit -l")
out["nproc"] = sh("nproc")
out["hugepages"] = sh("cat /proc/meminfo | head -20")
out["cgroup_mem"] = sh("cat /sys/fs/cgroup/memory.max 2>/dev/null; cat /sys/fs/cgroup/memory/memory.limit_in_bytes 2>/dev/null")
out["gpu_numa"] = sh("for d in /sys/bus/pci/devices/*; do c=$(cat $d/class 2>/dev/null); if [ \"$c\" = 0x030200 ]; then echo $d $(cat $d/numa_node); fi; done")

dev = torch.device("cuda:0")
torch.cuda.set_device(dev)
def bw_curve():
    res = []
    maxb = 1 << 30
    h = torch.empty(maxb, dtype=torch.uint8, pin_memory=True)
    h2 = torch.empty(maxb, dtype=torch.uint8, pin_memory=True)
    h.fill_(1); h2.fill_(2)
    d = torch.empty(maxb, dtype=torch.uint8, device=dev)
    d2 = torch.empty(maxb, dtype=torch.uint8, device=dev)
    s1 = torch.cuda.Stream(); s2 = torch.cuda.Stream()
    sizes = [1 << p for p in range(16, 31)]
    for sz in sizes:
        reps = max(3, min(200, (1 << 30) // sz))
        row = {"bytes": sz}
        for mode in ("h2d", "d2h", "duplex"):
            best = 0.0
            for trial in range(3):
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
                f0 = torch.cuda.Event(enable_timing=True); f1 = torch.cuda.Event(enable_timing=True)
                if mode in ("h2d", "duplex"):
                    e0.record(s1)
                    with torch.cuda.stream(s1):
                        for r in range(reps):
                            d[:sz].copy_(h[:sz], non_blocking=True)
                    e1.record(s1)
                if mode in ("d2h", "duplex"):
                    f0.record(s2)
                    with torch.cuda.stream(s2):
                        for r in range(reps):
                            h2[:sz].copy_(d2[:sz], non_blocking=True)
                    f1.record(s2)
                torch.cuda.synchronize()
                if mode == "h2d":
                    gbs = sz * reps / (e0.elapsed_time(e1) * 1e-3) / 1e9
                    best = max(best, gbs)
                elif mode == "d2h":
                    gbs = sz * reps / (f0.elapsed_time(f1) * 1e-3) / 1e9
                    best = max(best, gbs)
                else:
                    a = sz * reps / (e0.elapsed_time(e1) * 1e-3) / 1e9
                    b = sz * reps / (f0.elapsed_time(f1) * 1e-3) / 1e9
                    if (a + b) > best:
                        best = a + b; row["duplex_h2d"] = a; row["duplex_d2h"] = b
            row[mode] = best
        res.append(row)
        print(row, flush=True)
    # HBM copy
    torch.cuda.synchronize()
    best = 0
    for t in range(10):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); d2.copy_(d); e1.record(); torch.cuda.synchronize()
        best = max(best, 2 * maxb / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    return res, best

t0 = time.time()
curve, hbm = bw_curve()
out["link_curve"] = curve
out["hbm_copy_gbs"] = hbm
# pinned alloc speed
t = time.time(); x = torch.empty(8 << 30, dtype=torch.uint8, pin_memory=True); out["pin_8GiB_s"] = time.time() - t
del x
out["elapsed_s"] = time.time() - t0
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
print(json.dumps({k: v for k, v in out.items() if k not in ("link_curve", "lscpu", "topo", "hugepages")}, indent=1))
print(out["lscpu"][:1500])
