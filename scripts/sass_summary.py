"""SASS instruction summary of compiled kernels (cuobjdump -sass): mnemonic histogram per
cubin / shared object, plus the markers that show what the kernel uses on sm_100a (bulk async
copies UBLKCP, cp.async LDGSTS, FP64 DFMA/DMUL/DADD, warp shuffles SHFL, no tensor-core MMA).

    python scripts/sass_summary.py <file.cubin|libqgpu.so> [...] [--kernel NAME] [--top 25]
"""
import collections
import re
import subprocess
import sys


def sass(path):
    return subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", path], capture_output=True, text=True).stdout


def summarise(text, kernel=None):
    out = collections.OrderedDict()
    cur = None
    for line in text.splitlines():
        m = re.match(r"\s*Function : (\S+)", line)
        if m:
            cur = m.group(1)
            if kernel and kernel not in cur:
                cur = None
            else:
                out[cur] = collections.Counter()
            continue
        if cur is None:
            continue
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.[A-Z0-9_.]+)?", line)
        if m:
            out[cur][m.group(2)] += 1
    return out


def main():
    args = [a for a in sys.argv[1:]]
    kernel = args[args.index("--kernel") + 1] if "--kernel" in args else None
    top = int(args[args.index("--top") + 1]) if "--top" in args else 25
    files = [a for i, a in enumerate(args) if not a.startswith("--") and (i == 0 or args[i - 1] not in ("--kernel", "--top"))]
    marks = ["UBLKCP", "LDGSTS", "SYNCS", "DFMA", "DMUL", "DADD", "SHFL", "LDS", "STS", "STG", "LDG", "BAR",
             "HMMA", "UTCHMMA", "UTCQMMA", "DMMA"]
    for f in files:
        for fn, c in summarise(sass(f), kernel).items():
            tot = sum(c.values())
            print(f"{f} :: {fn}: {tot} SASS instructions")
            print("  markers: " + ", ".join(f"{k} {c.get(k, 0)}" for k in marks))
            print("  top: " + ", ".join(f"{k} {v}" for k, v in c.most_common(top)))


if __name__ == "__main__":
    main()
