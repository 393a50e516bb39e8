"""Quick timing of pt_mcmc on an MCMC config (diagnostic; bench.py --config m2 is the bench line)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import phantom
import paper_conf_ipps_xuzwrwxgxy12_b200 as pt

name = sys.argv[1] if len(sys.argv) > 1 else "m2"
d = phantom.mcmc_config(name)
tr = pt.Tracker(0)
dw = torch.as_tensor(d.dwi, device="cuda")
bv = torch.as_tensor(d.bvals, device="cuda")
bc = torch.as_tensor(d.bvecs, device="cuda")
mk = torch.as_tensor(d.mask, device="cuda")
dd = d.replace(dwi=dw, bvals=bv, bvecs=bc, mask=mk)
for rep in range(3):
    s, _ = tr.mcmc(dd)
    torch.cuda.synchronize()
    st = tr.mcmc_stats()
    print(name, "voxels", st["voxels"], "kernel_ms", round(st["kernel_ms"], 2),
          "voxels/s", round(st["voxels"] / st["kernel_ms"] * 1e3), "MH steps/s",
          "%.3g" % (st["mh_steps"] / st["kernel_ms"] * 1e3), "acc", round(st["accepted"] / st["mh_steps"], 3), flush=True)
