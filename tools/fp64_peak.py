"""Runs tools/ubench/fp64_peak (FP64 pipe peak) under an NVML clock sampler and writes
profiles/<tag>_fp64_peak.json — the measured FP64 peak bench.py's roofline "alu" view divides by.
usage: python tools/fp64_peak.py TAG"""
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tools", "ubench", "fp64_peak.cu")
EXE = os.path.join(ROOT, "tools", "ubench", "fp64_peak")


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r02"
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-o", EXE, SRC])
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(0)
    samples, reasons, stop = [], set(), threading.Event()

    def loop():
        while not stop.is_set():
            samples.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
            reasons.add(int(pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)))
            time.sleep(0.02)

    t = threading.Thread(target=loop, daemon=True)
    t.start()
    out = subprocess.run([EXE], capture_output=True, text=True, check=True).stdout
    stop.set(); t.join()
    lines = [json.loads(l) for l in out.splitlines() if l.startswith("{")]
    ops = {}
    for d in lines[1:]:
        o = ops.setdefault(d["op"], d)
        if d["lane_ops_per_s"] > o["lane_ops_per_s"]:
            ops[d["op"]] = d
    load = [s for s in samples if s > 500]
    maxmhz = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
    med = statistics.median(load) if load else maxmhz
    for o in ops.values():   # per-SM rate at the NVML clock (the pipe: 64 FP64 lanes/clk/SM)
        o["lane_ops_per_clk_per_sm_at_nvml_clock"] = o["lane_ops_per_s"] / (med * 1e6) / lines[0]["sms"]
    best = max(o["lane_ops_per_s"] for o in ops.values())
    res = {"what": "FP64 pipe peak on this B200 (tools/ubench/fp64_peak.cu): 16 independent chains per thread, "
                   "2 CTAs x 512 threads per SM, best of 2 runs per op; one DFMA/DADD/DMUL = one FP64 lane-op",
           "device": lines[0], "ops": ops,
           "peak_lane_ops_per_s": best,
           "peak_dfma_tflops": 2 * ops["dfma_uniform"]["lane_ops_per_s"] / 1e12,
           "nvml": {"sm_mhz_median_under_load": statistics.median(load) if load else None, "sm_max_mhz": maxmhz,
                    "samples": len(samples), "reason_bits_seen": sorted(reasons)},
           "nominal_at_max_clock": 148 * 64 * maxmhz * 1e6}
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    p = os.path.join(ROOT, "profiles", f"{tag}_fp64_peak.json")
    json.dump(res, open(p, "w"), indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
