"""Phase-0 probe: host facts and pinned host<->HBM bandwidth on one B200.

Measures H2D, D2H and concurrent duplex copies from pinned host memory with CUDA
events (best of several 1 GiB transfers in 128 MiB chunks). Prints one JSON line.
"""
import json, os, time, subprocess
import torch

def main():
    out = {}
    out["cpu_count"] = os.cpu_count()
    out["affinity"] = len(os.sched_getaffinity(0))
    with open("/proc/meminfo") as f:
        for line in f:
            if line.startswith(("MemTotal", "MemAvailable")):
                k, v = line.split(":")
                out[k] = v.strip()
    try:
        out["numa_nodes"] = sorted(os.listdir("/sys/devices/system/node"))
    except Exception as e:
        out["numa_nodes"] = str(e)
    p = torch.cuda.get_device_properties(0)
    out["gpu"] = p.name
    out["sms"] = p.multi_processor_count
    out["hbm_total"] = p.total_memory
    try:
        bus = subprocess.run(["nvidia-smi", "--query-gpu=pci.bus_id,pcie.link.gen.current,pcie.link.width.current,pcie.link.gen.max", "--format=csv,noheader"], capture_output=True, text=True).stdout
        out["pcie"] = bus.strip()
    except Exception as e:
        out["pcie"] = str(e)
    GiB = 1 << 30
    chunk = 128 << 20
    t0 = time.time()
    h_src = torch.empty(GiB, dtype=torch.uint8).pin_memory()
    h_dst = torch.empty(GiB, dtype=torch.uint8).pin_memory()
    out["pin_2GiB_s"] = time.time() - t0
    d = torch.empty(GiB, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(GiB, dtype=torch.uint8, device="cuda")
    s1 = torch.cuda.Stream(); s2 = torch.cuda.Stream()

    def run(mode):
        best = 0
        for _ in range(6):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            s1.wait_event(e0); s2.wait_event(e0)
            nbytes = 0
            for off in range(0, GiB, chunk):
                if mode in ("h2d", "duplex"):
                    with torch.cuda.stream(s1):
                        d[off:off+chunk].copy_(h_src[off:off+chunk], non_blocking=True)
                    nbytes += chunk
                if mode in ("d2h", "duplex"):
                    with torch.cuda.stream(s2):
                        h_dst[off:off+chunk].copy_(d2[off:off+chunk], non_blocking=True)
                    nbytes += chunk
            ev1 = torch.cuda.Event(); ev1.record(s1)
            ev2 = torch.cuda.Event(); ev2.record(s2)
            torch.cuda.current_stream().wait_event(ev1); torch.cuda.current_stream().wait_event(ev2)
            e1.record(); torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            best = max(best, nbytes / (ms * 1e-3) / 1e9)
        return best
    out["h2d_GBps"] = run("h2d")
    out["d2h_GBps"] = run("d2h")
    out["duplex_GBps"] = run("duplex")
    x = torch.empty(1 << 30, dtype=torch.bfloat16, device="cuda")
    y = torch.empty_like(x)
    for _ in range(3): y.copy_(x)
    torch.cuda.synchronize()
    e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
    e0.record(); [y.copy_(x) for _ in range(10)]; e1.record(); torch.cuda.synchronize()
    out["hbm_copy_GBps"] = 10 * 2 * x.numel() * 2 / (e0.elapsed_time(e1) * 1e-3) / 1e9
    print(json.dumps(out))

if __name__ == "__main__":
    main()
