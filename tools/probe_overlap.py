import sys, torch, json
sys.path.insert(0, '.')
import fieldgen
from paper_conf_sc_dufekgaad024_b200 import Dslash
torch.cuda.set_device(0)
dims = tuple(int(x) for x in sys.argv[1].split(','))
mask = int(sys.argv[2])
fat, lng = fieldgen.workload_links(dims)
from paper_conf_sc_dufekgaad024_b200 import _abi
for mode in ("none", "sites", "dirs", "fused"):
    for transport in ("nccl", "p2p", "dryrun"):
        tr = "nccl" if transport == "dryrun" else transport
        with Dslash(dims, parity_mask=0, force_halo=mask, overlap=mode, timing=True, transport=tr) as D:
            D.load_links(fat, lng)
            if transport == "dryrun":   # same stream structure, no bytes moved (timing only)
                _abi.dslash_set_option(D.h, _abi.DSLASH_OPT_HALO_DRYRUN, 1)
            srcs = [torch.from_numpy(fieldgen.vector_cb(dims, 3 + r, 1)).cuda() for r in range(4)]
            outs = [D.empty_vector() for _ in range(4)]
            for i in range(20): D.apply(outs[i % 4], srcs[i % 4], 0)
            torch.cuda.synchronize(); D.kernel_timing_reset()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            for i in range(200): D.apply(outs[i % 4], srcs[i % 4], 0)
            b.record(); torch.cuda.synchronize()
            res = {k: D.kernel_timing(k) for k in range(4)}
            print(mode, transport, "step_us %.1f" % (a.elapsed_time(b) / 200 * 1e3),
                  {k: ("%.1f us x %d" % (v[0] / max(1, v[1]) * 1e3, v[1])) for k, v in res.items()}, flush=True)
