"""Per-source-line instruction and stall shares of one kernel in an ncu report.

ncu's source page (SASS view, `--page source --print-source sass`) gives executed
warp instructions and stall samples per SASS instruction; nvdisasm -g of the
object the kernel was compiled from maps each SASS offset to a source line.
The object must be the same build the report was taken with.

    python tools/ncu_lines.py gpurun_out/ncu_x.ncu-rep build/obj/traverse.o bfs_expand_kernelILb0ELi0ELi3 [top]
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile


def main():
    rep, obj, fn = sys.argv[1:4]
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    data = [r for r in rows[2:] if len(r) == len(hdr)]
    ia = hdr.index("Instructions Executed")
    ss = hdr.index("Warp Stall Sampling (All Samples)")
    base = int(data[0][0], 16)
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
        cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
        sass = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
    lines = sass.split("\n")
    start = [i for i, ln in enumerate(lines) if ln.startswith("//--------------------- .text.") and fn in ln][0]
    where, cur = {}, None
    for ln in lines[start + 1:]:
        if ln.startswith("//--------------------- .text."):
            break
        m = re.match(r'\s*//## File "(.*)", line (\d+)', ln)
        if m:
            cur = (os.path.basename(m.group(1)), int(m.group(2)))
            continue
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+", ln)
        if m and cur:
            where[int(m.group(1), 16)] = cur
    inst, stall = collections.Counter(), collections.Counter()
    for r in data:
        k = where.get(int(r[0], 16) - base, ("?", 0))
        inst[k] += int(r[ia])
        stall[k] += int(r[ss])
    ti, ts = sum(inst.values()), sum(stall.values())
    print(f"{rep}: {ti} warp instructions, {ts} stall samples, {len(data)} SASS instructions, "
          f"{sum(1 for r in data if int(r[0], 16) - base in where)} mapped")
    for k, v in inst.most_common(top):
        print(f"  {k[0]:>26s}:{k[1]:<5d} inst {100 * v / ti:5.1f}%  stall {100 * stall[k] / ts:5.1f}%")


if __name__ == "__main__":
    main()
