"""Blackwell-path evidence from the built library (no GPU): per kernel, the
count of the SASS opcodes that show the sm_100a features the kernels use —
UBLKCP (1-D TMA bulk copies, both directions), SYNCS (mbarrier ops), STAS
(st.async), FADD2/FFMA2/FMUL2 (packed fp32), FHADD (fp32 + fp16 add), LDGSTS
(cp.async), STG.E.ENL2.256 (256-bit stores), REDUX (warp reductions) — from
cuobjdump -sass.  usage: python scripts/sass_summary.py > profiles/r02_sass_opcodes.json"""
import collections
import json
import re
import subprocess
import sys
from pathlib import Path

ROOT = Path(__file__).resolve().parent.parent
LIB = ROOT / "paper_conf_ipps_ibrahimo22_b200" / "libspp.so"
KEYS = ["UBLKCP", "SYNCS", "STAS", "FADD2", "FFMA2", "FMUL2", "FHADD", "LDGSTS", "STG.E.ENL2.256", "LDG.E.ENL2.256",
        "REDUX", "UTMACMDFLUSH", "F2FP", "PRMT", "BAR", "ELECT"]


def main():
    sass = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", str(LIB)], capture_output=True, text=True).stdout
    arch = sorted(set(re.findall(r"arch = (sm_\w+)", sass)))
    kernels = {}
    cur = None
    for line in sass.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            kernels[cur] = collections.Counter()
            continue
        m = re.match(r"\s+/\*[0-9a-f]+\*/\s+(@!?U?P\w+\s+)?([A-Z0-9_.]+)", line)
        if cur and m:
            op = m.group(2)
            for k in KEYS:
                if op == k or op.startswith(k + "."):
                    kernels[cur][k] += 1
            kernels[cur]["_total"] += 1
    short = {}
    for name, c in kernels.items():
        dem = subprocess.run(["c++filt"], input=name, capture_output=True, text=True).stdout.strip()
        short[dem[:160]] = dict(sorted(c.items()))
    json.dump({"library": str(LIB.relative_to(ROOT)), "arch": arch, "kernels": short}, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main()
