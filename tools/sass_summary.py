"""Per-kernel SASS instruction counts of libtg.so (cuobjdump -sass): the evidence that the
tensor-core units issue tcgen05 MMAs (UTCHMMA), TMEM loads/stores (LDTM/STTM), TMA tensor
loads (UTMALDG) and bulk copies (UBLKCP), and that the FP32 units run paired FMAs (FFMA2).
Usage: python tools/sass_summary.py [> profiles/rNN/sass_summary.txt]"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_sundaramrc09_b200", "libtg.so")
OPS = ["UTCHMMA", "UTCBAR", "LDTM", "STTM", "UTMALDG", "UBLKCP", "LDGSTS", "SYNCS", "FFMA2", "FFMA", "HMMA",
       "MUFU.EX2", "MUFU.RCP", "MUFU.TANH", "LDS.128", "STG.E.128"]


def short(mangled: str) -> str:
    try:
        d = subprocess.run(["c++filt", mangled], capture_output=True, text=True).stdout.strip()
    except OSError:
        d = mangled
    d = re.sub(r"\(anonymous namespace\)::", "", d)
    d = re.sub(r"\(.*\)$", "", d)
    return d.replace("tg::", "")


def main():
    sass = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True).stdout
    funcs = collections.OrderedDict()
    cur = None
    for line in sass.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = short(m.group(1))
            funcs.setdefault(cur, collections.Counter())
            continue
        if cur is None:
            continue
        m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]+)", line)
        if not m:
            continue
        ins = m.group(1)
        for op in OPS:
            if ins == op or ins.startswith(op + ".") or (op in ("LDS.128", "STG.E.128", "MUFU.EX2", "MUFU.RCP",
                                                                   "MUFU.TANH") and ins.startswith(op)):
                funcs[cur][op] += 1
                break
    print(f"# SASS instruction counts per kernel of {os.path.relpath(LIB, ROOT)} (cuobjdump -sass, sm_100a)")
    print("# kernel | " + " ".join(OPS))
    for f, c in funcs.items():
        if not any(c.values()):
            continue
        print(f"{f} | " + " ".join(f"{op}={c[op]}" for op in OPS if c[op]))
    tot = collections.Counter()
    for c in funcs.values():
        tot.update(c)
    print("# total | " + " ".join(f"{op}={tot[op]}" for op in OPS if tot[op]))


if __name__ == "__main__":
    sys.exit(main())
