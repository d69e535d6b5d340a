"""Interleaved A/B of the bench step (reset + circuit + 10^6 samples; host wall time, mean of 10)
across library builds.  usage: [AB_N=30 AB_D=14 AB_PIN=3 AB_T=12 AB_F=1 AB_WL=rqc|sycamore AB_BEAM=1..8] python tools/ab_step.py <rounds> <lib.so> ...
"""
import json, os, subprocess, sys
CHILD = r'''
import sys, time, json
sys.path.insert(0, "/root/repo")
import torch
import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W
import os
n=int(os.environ.get("AB_N", "30")); d=int(os.environ.get("AB_D", "14"))
h=sv.sv_create(n)
if os.environ.get("AB_PIN"): sv.sv_set_option(h, sv.SV_OPT_PASS_PIN, int(os.environ["AB_PIN"]))
if os.environ.get("AB_T"): sv.sv_set_blocking(h, int(os.environ["AB_T"]))
if os.environ.get("AB_BEAM"): sv.sv_set_option(h, sv.SV_OPT_PASS_SEARCH, int(os.environ["AB_BEAM"]))
F=int(os.environ.get("AB_F", "1"))
gates=W.sycamore_rqc(n,d) if os.environ.get("AB_WL")=="sycamore" else W.rqc(n,d)
c=sv.sv_circuit_create(h, gates, F)
out=torch.empty(1000000, dtype=torch.int64, device="cuda")
def step():
    sv.sv_reset(h); sv.sv_circuit_run_device(h,c); sv.sv_sample_device(h,1,1000000,out.data_ptr())
for _ in range(3): step()
sv.sv_synchronize(h)
t0=time.perf_counter()
for _ in range(10): step()
sv.sv_synchronize(h)
print(json.dumps({"step_ms": (time.perf_counter()-t0)/10*1e3, "passes": sv.sv_last_stats(h)["n_passes"]}))
'''
libs = sys.argv[2:]
for r in range(int(sys.argv[1])):
    for lib in libs:
        o = subprocess.run([sys.executable, "-c", CHILD], env=dict(os.environ, SVB200_LIB=lib), capture_output=True, text=True)
        print(os.path.basename(lib), o.stdout.strip()[-60:] or o.stderr[-300:], flush=True)
