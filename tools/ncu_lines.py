"""Per-source-line totals (instructions executed, stall samples) of one kernel launch in an
ncu report captured with --import-source on (uses the correlated cuda,sass source page).
usage: python tools/ncu_lines.py REPORT [launch_index] [top_n] [source_dir]
source_dir: where the NVRTC sources were dumped (PGVC_DUMP_SRC) to print the line text."""
import os
import csv
import io
import subprocess
import sys


def main(rep, idx=0, top=40, srcdir=None):
    texts = {}

    def text(f, n, fallback):
        if srcdir and os.path.exists(os.path.join(srcdir, f)):
            if f not in texts:
                texts[f] = open(os.path.join(srcdir, f)).read().split("\n")
            if 0 < n <= len(texts[f]):
                return texts[f][n - 1].strip()[:90]
        return fallback
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--launch-skip", str(idx), "--launch-count", "1"], capture_output=True, text=True).stdout
    agg, cur, path, hdr = {}, None, "", None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            path = r[1].rsplit("/", 1)[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None or len(r) < 8:
            continue
        if not r[0]:      # SASS rows: the source-line row above carries their totals
            continue
        cur = (path, int(r[0]), text(path, int(r[0]), r[1].strip()[:90]))
        num = lambda x: int(x) if x and x != "-" else 0
        ie, smp = num(r[7]), num(r[4])
        a = agg.setdefault(cur, [0, 0])
        a[0] += ie
        a[1] += smp
    ti = sum(a[0] for a in agg.values()) or 1
    ts = sum(a[1] for a in agg.values()) or 1
    print("instructions %d, samples %d" % (ti, ts))
    key = 1 if os.environ.get("SORT_SAMPLES") else 0
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1][key])[:top]:
        print("%6.2f%% ins %6.2f%% smp  %s:%d  %s" % (100 * a[0] / ti, 100 * a[1] / ts, k[0], k[1], k[2]))


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0, int(sys.argv[3]) if len(sys.argv) > 3 else 40,
         sys.argv[4] if len(sys.argv) > 4 else None)
