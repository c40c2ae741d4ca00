"""Per-source-line shared-memory wavefronts (and excess from bank conflicts) of one ncu --set full
capture, joined with the SASS line table of the kernel's cubin (run here, no GPU).

  python tools/ncu_lines.py gpurun_out/prof_iter.ncu-rep paper_conf_sc_antepara0jh24_b200/build/sweep2p.cu.o 'sweep2p_kernelILj0E'
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile


def main(rep, obj, kname):
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=tmp, capture_output=True)
    cub = [f for f in os.listdir(tmp) if f.endswith(".cubin")][0]
    sass = subprocess.run(["nvdisasm", "-g", os.path.join(tmp, cub)], capture_output=True, text=True).stdout.split("\n")
    start = next(i for i, l in enumerate(sass) if l.startswith(".text.") and kname in l)
    pc2line, cur = {}, None
    for l in sass[start + 1:]:
        if l.startswith(".text.") or re.match(r"\s*\.section", l):
            break
        m = re.search(r'File "(.*?)", line (\d+)', l)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m2 = re.search(r"/\*([0-9a-f]{4,})\*/\s+(.*?);", l)
        if m2:
            pc2line[int(m2.group(1), 16)] = cur
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(k for k in range(3) if "Address" in rows[k])
    h = rows[hi]
    ix = {n: i for i, n in enumerate(h)}
    data = [r for r in rows[hi + 1:] if len(r) == len(h)]
    base = min(int(r[ix["Address"]], 16) for r in data)
    wav, exc, ops = collections.Counter(), collections.Counter(), collections.defaultdict(set)
    for r in data:
        w = float(r[ix["L1 Wavefronts Shared"]] or 0)
        if w == 0:
            continue
        k = pc2line.get(int(r[ix["Address"]], 16) - base)
        wav[k] += w
        exc[k] += float(r[ix["L1 Wavefronts Shared Excessive"]] or 0)
        ops[k].add(r[ix["Source"]].split()[0] if not r[ix["Source"]].strip().startswith("@") else r[ix["Source"]].split()[1])
    tot = sum(wav.values())
    print(f"total shared wavefronts {tot:.4g}, excessive {sum(exc.values()):.4g}")
    for k, v in wav.most_common():
        print(f"{str(k):32s} {v:12.0f} {exc[k]:12.0f} {100 * v / tot:5.1f}%  {','.join(sorted(ops[k]))}")


if __name__ == "__main__":
    main(*sys.argv[1:4])
