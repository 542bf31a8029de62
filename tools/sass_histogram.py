"""SASS opcode histogram of libirr.so (cuobjdump -sass), per kernel and in
total: the evidence of which pipes the kernels use (DMMA = FP64 tensor core
via mma.sync; DFMA = FP64 FMA pipe; LDGSTS = cp.async; UTMALDG / UBLKCP =
TMA; REDUX / SHFL = warp reductions).

    python tools/sass_histogram.py [lib.so] [--kernels]
"""
import collections
import re
import subprocess
import sys

lib = sys.argv[1] if len(sys.argv) > 1 and not sys.argv[1].startswith("--") else \
    "paper_conf_sc_abdelfattahgbtld22_b200/libirr.so"
out = subprocess.run(["cuobjdump", "-sass", lib], capture_output=True, text=True).stdout
FOCUS = ("DMMA", "DFMA", "DMUL", "DADD", "MUFU", "LDGSTS", "UTMALDG", "UTMASTG", "UBLKCP", "LDG", "STG", "LDS",
         "STS", "SHFL", "CREDUX", "REDUX", "BAR", "RED", "REDG", "ATOMG", "HMMA", "UTCHMMA")
total = collections.Counter()
per = collections.defaultdict(collections.Counter)
func = None
for line in out.splitlines():
    m = re.match(r"\s+Function : (\S+)", line)
    if m:
        func = m.group(1)
        continue
    m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]+)?", line)
    if m and func:
        op = m.group(1)
        total[op] += 1
        per[func][op] += 1
print(f"# SASS opcode histogram of {lib} (cuobjdump -sass), {sum(total.values())} instructions, "
      f"{len(per)} kernels")
print("# focus opcodes (whole library):")
for op in FOCUS:
    print(f"{op:10s} {total.get(op, 0):7d}")
if "--kernels" in sys.argv:
    print("# per kernel (focus opcodes > 0):")
    for f, c in sorted(per.items(), key=lambda kv: -sum(kv[1].values())):
        pretty = subprocess.run(["c++filt", f], capture_output=True, text=True).stdout.strip()[:110]
        focus = {op: c[op] for op in FOCUS if c.get(op)}
        print(f"{pretty}\n    {sum(c.values())} instr  {focus}")
