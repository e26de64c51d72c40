"""Probe the GPU box: host RAM/CPU, PCIe pinned-copy bandwidth (H2D, D2H, both), HBM copy."""
import os, subprocess, json, time, torch
out = {}
out["nproc"] = os.cpu_count()
out["meminfo"] = open("/proc/meminfo").read().split("\n")[:3]
out["lscpu"] = subprocess.run("lscpu | head -20", shell=True, capture_output=True, text=True).stdout
out["smi"] = subprocess.run("nvidia-smi; nvidia-smi topo -m; nvidia-smi -q | grep -i -A3 'PCIe Generation\\|Link Width'", shell=True, capture_output=True, text=True).stdout
out["shm"] = subprocess.run("df -h /dev/shm; cat /proc/sys/vm/nr_hugepages; ulimit -l", shell=True, capture_output=True, text=True).stdout
dev = torch.device("cuda:0")
def bw(fn, nbytes, it=10):
    s, e = torch.cuda.Event(True), torch.cuda.Event(True)
    fn(); torch.cuda.synchronize()
    best = 1e9
    for _ in range(it):
        s.record(); fn(); e.record(); e.synchronize(); best = min(best, s.elapsed_time(e))
    return nbytes / best / 1e6
n = 1 << 30
h = torch.empty(n, dtype=torch.uint8, pin_memory=True)
d = torch.empty(n, dtype=torch.uint8, device=dev)
d2 = torch.empty(n, dtype=torch.uint8, device=dev)
out["h2d_gbs"] = bw(lambda: d.copy_(h, non_blocking=True), n)
out["d2h_gbs"] = bw(lambda: h.copy_(d, non_blocking=True), n)
s2 = torch.cuda.Stream()
h2 = torch.empty(n, dtype=torch.uint8, pin_memory=True)
def both():
    d.copy_(h, non_blocking=True)
    with torch.cuda.stream(s2):
        h2.copy_(d2, non_blocking=True)
    torch.cuda.current_stream().wait_stream(s2)
out["bidir_gbs"] = bw(both, 2 * n)
out["hbm_copy_gbs"] = bw(lambda: d2.copy_(d), 2 * n)
t0 = time.time(); x = torch.empty(8 << 30, dtype=torch.uint8, pin_memory=True); out["pin_8g_s"] = time.time() - t0
print(json.dumps(out, indent=1))
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/probe.json", "w"), indent=1)
