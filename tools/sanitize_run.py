"""Small applies through every kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck).  python tools/sanitize_run.py  -> exits 0 if every result matches."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np
import torch

import fieldgen
from paper_conf_sc_dufekgaad024_b200 import Dslash

torch.cuda.set_device(0)
dims = (16, 8, 8, 8)
fat, lng = fieldgen.workload_links(dims)
src = {p: torch.from_numpy(fieldgen.vector_cb(dims, 3, p)).cuda() for p in (0, 1)}
ref = None
cases = [dict(kernel=k) for k in ("site", "dir2", "dir4")]
cases += [dict(force_halo=m, overlap=ov) for m in (0x8, 0xC) for ov in (True, False)]
cases += [dict(force_halo=0xC, transport="p2p"), dict(recon=12), dict(precision="mixed"), dict(pdl=False)]
# later additions: the neighbour-staged kernel (TMA bulk copies + mbarrier into shared memory), the
# split-by-direction overlap, NCCL to self,
# and the mixed-precision CG (fp32 links converted from the fp64 ones)
cases += [dict(stage=True), dict(stage=True, kernel="site", force_halo=0xC), dict(stage=True, precision="f32"),
          dict(force_halo=0xC, overlap="dirs"), dict(force_halo=0xC, overlap="dirs", precision="f32"),
          dict(force_halo=0xC, self_nccl=True), dict(cg_mixed=True)]
# third session: the producer push (stencil epilogue and CG direction update store into the
# peer-mapped ghost bank; flag waits/writes on the streams) and recon-9 long links
cases += [dict(force_halo=0xC, transport="p2p", push=True), dict(force_halo=0x8, transport="p2p", push=True, overlap="dirs"),
          dict(recon=9), dict(recon=9, kernel="site", force_halo=0xC), dict(recon=9, stage=True)]
n = 0
for kw in cases:
    kw = dict(kw)
    mixed_cg = kw.pop("cg_mixed", False)
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        if mixed_cg:
            x = D.empty_vector()
            D.cg_mixed(x, src[0], 0, 0.5, rel_tol=1e-8, inner_tol=1e-2, max_iter=100)
        out = D.empty_vector()
        (D.apply_push if kw.get("push") else D.apply)(out, src[1].to(D.dtype), 0)
        o2 = D.empty_vector()
        D.apply(o2, out.to(D.dtype), 1)
        multi = torch.stack([src[1], src[1]]).to(D.dtype)
        mo = torch.empty_like(multi)
        D.apply_multi(mo, multi, 0)
        if D.precision != "f32":
            x = D.empty_vector()
            D.cg(x, src[0], 0, 0.5, rel_tol=1e-8, max_iter=50)
        torch.cuda.synchronize()
        r = out.cpu().numpy().astype(np.complex128)
        if ref is None:
            ref = r
        tol = 1e-5 if kw.get("precision") in ("mixed", "f32") else 1e-12
        err = np.abs(r - ref).max() / np.abs(ref).max()
        assert err <= tol, (kw, err)
        assert torch.equal(mo[0], mo[1])
        n += 1
# round 3: the site-blocked multi-RHS layout (conversion kernels + the VBLK stencil), 8 RHS
for kw in (dict(kernel="site"), dict(kernel="dir2"), dict(precision="f32", kernel="site"),
           dict(precision="mixed", kernel="site", recon=12), dict(recon=9, kernel="site")):
    with Dslash(dims, **kw) as D:
        D.load_links(fat, lng)
        multi = torch.stack([src[1] * (k + 1) for k in range(8)]).to(D.dtype).contiguous()
        planar = D.apply_multi(torch.empty_like(multi), multi, 0)
        bout = D.apply_multi_blocked(torch.empty_like(multi), D.to_blocked(torch.empty_like(multi), multi), 0)
        back = D.from_blocked(torch.empty_like(multi), bout)
        torch.cuda.synchronize()
        assert torch.equal(back, planar), kw
        n += 1
print(f"sanitize_run: {n} configurations OK")
