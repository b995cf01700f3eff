import os, sys, numpy as np
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
import paper_conf_ppopp_qawasmehchc15_b200 as seis
from paper_conf_ppopp_qawasmehchc15_b200 import inputs
def run(flag, nx, ny, nz, nb, nt):
    os.environ["SEIS_AC_STEP"] = flag
    m = inputs.random_media((nz, ny, nx), seed=61)
    w = inputs.source_series("acoustic", nt, 5e-4, 35.0)
    src = (min(128, nx - 1), min(14, ny - 1), nz // 2)
    rec = np.asarray([[0,0,0]], np.int32)
    g = seis.Grid(nx, ny, nz, 10.0, 5e-4, nb=nb, pml_f=35.0)
    mod = seis.Model(g, "acoustic", m["vp"], rho=m["rho"])
    sg = np.zeros((nt, 1), np.float32)
    mod.forward_model(seis.Shot(src, w, rec), sg)
    f = [mod.get_field(t) for t in range(4)]
    mod.close()
    return f
for (nx,ny,nz,nb) in [(150,45,120,7),(150,45,120,0),(128,14,50,0),(260,60,40,0)]:
  for nt in (1,2,3,5,37):
    a = run("0", nx,ny,nz,nb,nt); b = run("1", nx,ny,nz,nb,nt)
    out=[]
    for t in range(4):
        d = np.argwhere(a[t] != b[t])
        out.append((len(d), d[:3].tolist(), float(np.abs(a[t]-b[t]).max())))
    print((nx,ny,nz,nb), nt, out, flush=True)
