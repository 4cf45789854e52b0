"""Static code evidence for the stencil kernels (no GPU needed): the ptxas register / spill /
shared-memory table of every instantiation in one translation unit, and SASS instruction
counts + an excerpt of the default kernel and of the neighbour-staged kernel (UBLKCP = the
cp.async.bulk copy, SYNCS = the mbarrier operations).

    python tools/sass_report.py [kernels_f64_r18] > profiles/r02/sass_f64_r18.txt
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "paper_conf_sc_dufekgaad024_b200"))
import build  # noqa: E402

TU = sys.argv[1] if len(sys.argv) > 1 else "kernels_f64_r18"
src = os.path.join(ROOT, "paper_conf_sc_dufekgaad024_b200", "csrc", TU + ".cu")
obj = f"/tmp/{TU}_report.o"
cmd = ["nvcc", *build.ARCH, "-lineinfo", "-O3", "-std=c++17", "-Xcompiler", "-fPIC", "-I",
       os.path.join(build.nccl_dir(), "include"), "-I", os.path.join(ROOT, "include"), "-Xptxas", "-v", "-c", src,
       "-o", obj]
r = subprocess.run(cmd, capture_output=True, text=True, check=True)


def demangle(names):
    out = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True).stdout.split("\n")
    return dict(zip(names, out))


# ---- ptxas table
rows, cur = [], None
for line in r.stderr.splitlines():
    m = re.search(r"Compiling entry function '(\w+)'", line)
    if m:
        cur = {"name": m.group(1)}
        rows.append(cur)
        continue
    if cur is None:
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m:
        cur["stack"], cur["spill_st"], cur["spill_ld"] = map(int, m.groups())
    m = re.search(r"Used (\d+) registers", line)
    if m:
        cur["regs"] = int(m.group(1))
    m = re.search(r"(\d+) bytes smem", line)
    if m:
        cur["smem"] = int(m.group(1))
dm = demangle([x["name"] for x in rows])
print(f"# ptxas -v of csrc/{TU}.cu for sm_100a ({len(rows)} entry functions)")
print("# template args: dslash_kernel<LR, VR, LANES, GHOST, MINB, RECON, NRHS, RHSL>, "
      "dslash_stage_kernel<LR, VR, LANES, GHOST, RECON, NRHS, RHSL>")
print(f"{'regs':>5} {'stack':>6} {'spill_st':>9} {'spill_ld':>9} {'smem':>6}  kernel")
for x in sorted(rows, key=lambda x: dm[x["name"]]):
    n = dm[x["name"]].replace("(hisq::StencilParams)", "").replace("hisq::", "")
    print(f"{x.get('regs', 0):>5} {x.get('stack', 0):>6} {x.get('spill_st', 0):>9} {x.get('spill_ld', 0):>9} "
          f"{x.get('smem', 0):>6}  {n}")

# ---- SASS
sass = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True, check=True).stdout
funcs = re.split(r"\n\s+Function : ", sass)[1:]
by_name = {}
for f in funcs:
    name, body = f.split("\n", 1)
    by_name[name.strip()] = body


def opcode_hist(body):
    ops = collections.Counter()
    for line in body.splitlines():
        m = re.match(r"\s+/\*[0-9a-f]{4}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", line)
        if m:
            ops[m.group(1)] += 1
    return ops


def pick(pattern):
    for k in by_name:
        if re.search(pattern, demangle([k])[k]):
            return k
    return None


for title, pat in (("default kernel (dir2, fp64, recon 18, interior, MINB 2, 1 RHS)",
                    r"dslash_kernel<double, double, 2, false, 2, 18, 1, 1>"),
                   ("neighbour-staged kernel (site, fp64, recon 18, 1 RHS)",
                    r"dslash_stage_kernel<double, double, 1, false, 18, 1, 1>")):
    k = pick(re.escape(pat))
    if not k:
        print(f"\n# {title}: not found")
        continue
    ops = opcode_hist(by_name[k])
    print(f"\n# SASS of {title}: {demangle([k])[k]}")
    print("# instruction counts (static):")
    keys = [o for o in ops if re.match(r"(LDG|STG|LDS|UBLKCP|SYNCS|DFMA|DADD|DMUL|SHFL|ACQBULK|FENCE|CCTL|BAR|"
                                       r"UTMA|LDGSTS)", o)]
    for o in sorted(keys):
        print(f"  {o:<40} {ops[o]}")
    print(f"  total instructions {sum(ops.values())}")
    lines = [l for l in by_name[k].splitlines() if re.search(r"LDG|UBLKCP|SYNCS|STG|DFMA", l)]
    print("# excerpt (first 24 memory / fp64 instructions):")
    for l in lines[:24]:
        print("  " + re.sub(r"\s+/\* 0x[0-9a-f]+ \*/", "", l.strip()))
os.remove(obj)
