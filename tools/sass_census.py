"""SASS opcode census of the shipped kernels (cuobjdump -sass of build/obj/*.cu.o):

    python tools/sass_census.py > profiles/r02/sass_grep.txt

Counts, per kernel, the opcodes that prove the Blackwell path: UTCHMMA (tcgen05.mma), UTMALDG /
UTMASTG (TMA tensor load / store), UBLKCP (1-D bulk copy), LDTM / STTM (tcgen05.ld / st), UTCBAR
(tcgen05.commit), SYNCS (mbarrier), HMMA (mma.sync), LDSM (ldmatrix), FMNMX3, MUFU."""
import collections
import glob
import os
import re
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OPS = ["UTCHMMA", "UTMALDG", "UTMASTG", "UBLKCP", "LDTM", "STTM", "UTCBAR", "SYNCS", "HMMA", "LDSM", "FMNMX3",
       "MUFU", "UTCATOMSWS", "UTMACCTL"]


def main():
    print("# SASS opcode counts per kernel (cuobjdump -sass of build/obj/*.cu.o, libgllm.so's objects; sm_100a).")
    print("# UTCHMMA = tcgen05.mma, UTMALDG / UTMASTG = TMA tensor load / store, UBLKCP = cp.async.bulk, "
          "LDTM/STTM = tcgen05.ld/st, UTCBAR = tcgen05.commit, HMMA = mma.sync, LDSM = ldmatrix.")
    for obj in sorted(glob.glob(os.path.join(ROOT, "build", "obj", "*.cu.o"))):
        out = subprocess.run(["cuobjdump", "-sass", obj], capture_output=True, text=True).stdout
        print(f"== build/obj/{os.path.basename(obj)}")
        fn, cnt = None, collections.Counter()

        def flush():
            if fn and cnt:
                for op in OPS:
                    if cnt[op]:
                        print(f"{fn} {op} {cnt[op]}")
        for line in out.splitlines():
            m = re.match(r"\s+Function : (\S+)", line)
            if m:
                flush()
                fn = subprocess.run(["c++filt", m.group(1)], capture_output=True, text=True).stdout.strip()
                k = re.search(r"(\w+_kernel(<[^(]*>)?)", fn)
                fn = k.group(1) if k else fn[:60]
                cnt = collections.Counter()
                continue
            m = re.search(r"/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9]*)", line)
            if m:
                cnt[m.group(1)] += 1
        flush()


if __name__ == "__main__":
    main()
