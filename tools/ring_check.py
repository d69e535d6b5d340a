import sys, os; sys.path.insert(0,'/root/repo')
import numpy as np
import paper_conf_sc_markidis23_b200 as sv
from oracle import ref_c
from oracle import sv as osv
from workloads import rqc as W
for n, d, F, T, lazy in [(16,8,1,10,False),(16,8,1,10,True),(20,10,1,12,False),(20,10,2,13,True),(22,12,1,13,False)]:
    gates = W.rqc(n, d, seed=n)
    h = sv.sv_create(n); sv.sv_set_blocking(h, T)
    if not lazy: sv.sv_device_ptr(h)
    st = sv.sv_run_circuit(h, gates, F)
    got = sv.sv_get_state(h, n).astype(np.complex128); sv.sv_destroy(h)
    ref = ref_c.run(n, gates)
    print(n, d, F, T, lazy, 'passes', st['n_passes'], 'jit', st['n_jit_passes'], 'fid', osv.fidelity(got, ref), 'err/bound', np.abs(got-ref).max()/osv.max_abs_bound(n,d), flush=True)
