"""SASS evidence for profiles/: per kernel instance of the built sm_100a objects, counts of the
instructions that prove the FP64 tensor path (DMMA), the TMA pipeline (UTMALDG, SYNCS mbarrier
ops), cp.async (LDGSTS), spills (LDL/STL) and the epilogue's load/store order, plus a DMMA-loop
excerpt.  usage: python tools/sass_evidence.py > profiles/r02_sass_evidence.txt"""
import collections
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OBJ = os.path.join(ROOT, "paper_conf_sc_gautierl21_b200", "build")
KEEP = ("DMMA", "UTMALDG", "UTMACCTL", "SYNCS", "LDGSTS", "LDL", "STL", "ATOMS", "FENCE", "LDG.E.64", "STG.E.64")
for obj, want in (("dgemm_tma.cu.o", "dgemm_tma_kernel"), ("trxm_tile.cu.o", "trxm_base_kernel")):
    out = subprocess.run(["cuobjdump", "-sass", os.path.join(OBJ, obj)], capture_output=True, text=True).stdout
    print("===== %s: cuobjdump -sass (nvcc 12.9, -gencode arch=compute_100a,code=sm_100a -O3)" % obj)
    excerpt_done = False
    for f in re.split(r"\n\s+Function : ", out)[1:]:
        name = f.split("\n", 1)[0].strip()
        if want not in name:
            continue
        ops = [re.sub(r"^\s*/\*[0-9a-f]+\*/\s*", "", l).split(";")[0].strip() for l in f.splitlines() if re.match(r"\s*/\*[0-9a-f]{4}\*/", l)]
        c = collections.Counter()
        for o in ops:
            m = o.lstrip("@!PU0123456789T ").split(" ")[0] if o else ""
            m = re.sub(r"^@!?U?P\w+\s+", "", o).split(" ")[0]
            if any(m.startswith(k) for k in KEEP):
                c[m] += 1
        print("-- " + name)
        print("   " + ", ".join("%s x%d" % kv for kv in sorted(c.items())))
        if want == "dgemm_tma_kernel":
            seq = "".join("L" if "LDG.E.64" in o else "S" for o in ops if "LDG.E.64" in o or "STG.E.64" in o)
            print("   epilogue global load (L) / store (S) order: " + seq)
        if not excerpt_done:
            i = next(k for k, o in enumerate(ops) if "DMMA" in o or "LDGSTS" in o)
            print("   excerpt:")
            for o in ops[i:i + 24]:
                print("     " + o)
            excerpt_done = True
