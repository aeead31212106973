"""Probe: can NVML GPM (GPU Performance Monitoring, nvmlGpmMetricsGet) measure the
DRAM bandwidth of a timed region without a profiler?  Calibrates DRAM_BW_UTIL
against copies of known bytes, then reads it around C2 search steps."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pynvml as nv  # noqa: E402
import torch  # noqa: E402

nv.nvmlInit()
h = nv.nvmlDeviceGetHandleByIndex(0)
out = {}
try:
    sup = nv.nvmlGpmQueryDeviceSupport(h)
    out["gpm_supported"] = int(sup.isSupportedDevice)
except Exception as ex:  # noqa: BLE001
    out["gpm_supported_err"] = repr(ex)
print(json.dumps(out), flush=True)

METRICS = {"dram_bw_util": nv.NVML_GPM_METRIC_DRAM_BW_UTIL, "sm_util": nv.NVML_GPM_METRIC_SM_UTIL,
           "sm_occ": nv.NVML_GPM_METRIC_SM_OCCUPANCY}


def gpm(fn):
    s1, s2 = nv.nvmlGpmSampleAlloc(), nv.nvmlGpmSampleAlloc()
    torch.cuda.synchronize()
    nv.nvmlGpmSampleGet(h, s1)
    t0 = time.perf_counter()
    dev_s = fn()
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    nv.nvmlGpmSampleGet(h, s2)
    mg = nv.c_nvmlGpmMetricsGet_t()
    mg.version = nv.NVML_GPM_METRICS_GET_VERSION
    mg.numMetrics = len(METRICS)
    mg.sample1, mg.sample2 = s1, s2
    for i, m in enumerate(METRICS.values()):
        mg.metrics[i].metricId = m
    nv.nvmlGpmMetricsGet(mg)
    r = {k: mg.metrics[i].value for i, k in enumerate(METRICS)}
    nv.nvmlGpmSampleFree(s1)
    nv.nvmlGpmSampleFree(s2)
    r["wall_s"] = t1 - t0
    r["dev_s"] = dev_s
    return r


def timed(body):
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    body()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / 1e3


a = torch.empty(1 << 30, dtype=torch.float32, device="cuda")
b = torch.empty_like(a)
a.fill_(1.0)
for reps in (5, 20, 60):
    r = gpm(lambda: timed(lambda: [b.copy_(a) for _ in range(reps)]))
    byts = reps * 2 * a.numel() * 4
    r["GBps_events"] = byts / r["dev_s"] / 1e9
    r["implied_peak_GBps"] = r["GBps_events"] / max(r["dram_bw_util"], 1e-9) * 100
    r["bytes"] = byts
    print(json.dumps({"copy": reps, **r}), flush=True)
# read-only
for reps in (20,):
    r = gpm(lambda: timed(lambda: [a.sum() for _ in range(reps)]))
    byts = reps * a.numel() * 4
    r["GBps_events"] = byts / r["dev_s"] / 1e9
    r["implied_peak_GBps"] = r["GBps_events"] / max(r["dram_bw_util"], 1e-9) * 100
    print(json.dumps({"sum": reps, **r}), flush=True)
# idle gap inside the window: does util scale with active time?
r = gpm(lambda: (timed(lambda: [b.copy_(a) for _ in range(20)]), time.sleep(0.5))[0])
r["GBps_events"] = 20 * 2 * a.numel() * 4 / r["dev_s"] / 1e9
print(json.dumps({"copy_then_idle_0.5s": 20, **r}), flush=True)
del a, b
torch.cuda.empty_cache()

# C2 search steps
import ganns_synth as syn  # noqa: E402
import paper_conf_icde_yuwzqzl22_b200 as g  # noqa: E402
from bench import BenchIndex, Pipeline, make_workload  # noqa: E402

cfg = syn.CONFIGS["C2"]
X, Qs = make_workload(cfg, 0, 4)
Xd = torch.from_numpy(X).cuda()
Qds = [torch.from_numpy(q).cuda() for q in Qs]
idx = BenchIndex(g, cfg, Xd, 128, 64)
pipe = Pipeline(torch, idx, Qds, cfg.k, 2)
pipe.run(8, 128, 109)
ids, dists, st = idx.search(torch.cat(Qds), cfg.k, 128, e=109, stats=True)
st = st.long()
alg = int((4 * cfg.d + 4 * cfg.degree * st[:, 0] + 4 * cfg.d * st[:, 1]).sum()) // 4
for steps in (20, 100, 300):
    r = gpm(lambda: pipe.run(steps, 128, 109))
    r["ms_per_step"] = r["dev_s"] / steps * 1e3
    r["alg_GBps"] = alg / (r["dev_s"] / steps) / 1e9
    print(json.dumps({"c2_steps": steps, **r}), flush=True)
