import sys; sys.path.insert(0,'.')
import numpy as np
import paper_conf_sc_markidis23_b200 as sv
from workloads import rqc as W
n=30
h=sv.sv_create(n); sv.sv_device_ptr(h); sv.sv_set_timing(h, True)
qs=[11,17,21,23,25,26,27,28,29]
gates=[W.Gate(i,"h",(q,),W.GATE_H) for i,q in enumerate(qs)]
c=sv.sv_circuit_create(h,gates,1)
for _ in range(3):
    sv.sv_circuit_run_device(h,c); print(sv.sv_last_stats(h)["t_apply_high_dev_s"], flush=True)
