"""SASS instruction histogram of the kernels each bench workload times (the
labelled OC's default setting), from the NVRTC cubins the plans compile.

  python scripts/sass_histogram.py > profiles/r02_sass_histogram.md

Proves how the hand-written templates lower on sm_100a: UTMALDG (TMA tensor
loads), SYNCS (mbarrier ops), LDGSTS (cp.async), LDS/STS (shared), DFMA/FFMA.
Static counts (instructions in the binary), not dynamic ones. Host only.
"""
import collections
import glob
import os
import re
import subprocess
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

CASES = [  # (workload, stencil, dims, dtype, OC the round-2 bench labels)
    ("C2", "heat3d", (512, 512, 512), "f64", "ST_TB_BM_RT_PR"),
    ("C2", "heat3d", (512, 512, 512), "f64", "ST_RT_PR"),
    ("C3", "star25", (768, 768, 768), "f32", "ST_CM_RT_PR"),
    ("C4", "box125", (512, 512, 512), "f64", "ST_CM_RT_PR"),
    ("C5", "random3d:1:0", (1024, 1024, 1024), "f64", "ST_TB_BM_RT_PR"),
    ("C5", "random3d:2:4", (1024, 1024, 1024), "f64", "ST_BM_RT_PR"),
    ("C5", "random3d:3:8", (1024, 1024, 1024), "f64", "ST_BM_RT_PR"),
    ("C5", "random3d:4:12", (1024, 1024, 1024), "f64", "ST_BM_RT_PR"),
    ("N2", "random2d:1:0", (8192, 8192), "f64", "TB_BM"),
    ("N2", "random2d:2:4", (8192, 8192), "f64", "TB_BM"),
    ("N2", "random2d:3:8", (8192, 8192), "f64", "ST_BM_RT_PR"),
    ("unaligned rows", "edge:asym3d", (64, 64, 67), "f64", "ST_TB_BM_RT_PR"),
]
KEYS = ["UTMALDG", "UTMASTG", "UBLKCP", "LDGSTS", "SYNCS", "BAR", "LDS", "STS", "LDG", "STG", "SHFL", "DFMA",
        "DADD", "DMUL", "FFMA", "FFMA2", "UMOV", "LDCU", "IMAD", "IADD3", "BRA", "USETMAXREG"]


def main():
    import paper_conf_ipps_sunlyjlq22_b200 as sm
    import stencil_inputs as si
    print("# SASS instruction histograms of the timed kernels (static counts)\n")
    print("`python scripts/sass_histogram.py`: each plan's NVRTC cubin (sm_100a, `-lineinfo`) through "
          "`cuobjdump -sass`. Opcodes are counted by mnemonic (suffixes stripped).\n")
    print("| workload | stencil | OC | kernel | " + " | ".join(KEYS) + " | total |")
    print("|" + "---|" * (len(KEYS) + 5))
    for wl, name, dims, dtype, oc in CASES:
        d = tempfile.mkdtemp(prefix="sass_")
        os.environ["STENCIL_CACHE_DIR"] = d
        acc, c = si.config_stencil(name)
        p = sm.Plan(dims, acc, c, dtype, sm.oc_from_name(oc))
        low = p.info["kernel_name"]
        split = p.info["reg_split"][0] > 0
        sass = None
        for f in sorted(glob.glob(os.path.join(d, "*.name"))):   # the register-split check compiles
            if open(f).read() != low:                             # an unsplit twin with the same name
                continue
            txt = subprocess.run(["cuobjdump", "-sass", f[:-5] + ".cubin"], capture_output=True, text=True).stdout
            if sass is None or (("SETMAXREG" in txt) == split):
                sass = txt
        cnt = collections.Counter()
        for line in sass.splitlines():
            m = re.match(r"\s*/\*[0-9a-f]+\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)", line)
            if m:
                cnt[m.group(1)] += 1
        tot = sum(cnt.values())
        kname = re.sub(r"_ZN5smart\d+", "", low)[:40]
        m = re.match(r"_ZN5smart(\d+)", low)
        if m:
            n = int(m.group(1))
            kname = low[m.end():m.end() + n] + "<" + ",".join(re.findall(r"L[ib](\d+)E", low[m.end() + n:])) + ">"
        row = [str(cnt.get(k, 0)) for k in KEYS]
        print(f"| {wl} | {name} | {oc} | `{kname}` | " + " | ".join(row) + f" | {tot} |")
    print("\nUTMALDG = `cp.async.bulk.tensor` (TMA), SYNCS = mbarrier arrive/wait/try_wait, LDGSTS = "
          "`cp.async` (the unaligned-row staging), USETMAXREG = `setmaxnreg` (register split).")


if __name__ == "__main__":
    main()
