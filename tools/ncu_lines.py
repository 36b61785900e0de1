"""Per CUDA-source-line instruction and stall totals of one kernel (ncu --print-source cuda,sass)."""
import csv
import subprocess
import sys


def main(path, kregex, top=40):
    out = subprocess.run(['ncu', '-i', path, '--page', 'source', '--csv', '-k', f'regex:{kregex}', '--launch-count', '1',
                          '--print-source', 'cuda,sass'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hi = [i for i, r in enumerate(rows) if r and r[0] == 'Line No'][0]
    h = rows[hi]
    ii = h.index('Instructions Executed')
    wi = h.index('Warp Stall Sampling (All Samples)')
    lines = []
    for r in rows[hi + 1:]:
        if r and r[0] and len(r) > max(ii, wi):  # a source line row (aggregated)
            try:
                lines.append((float(r[ii] or 0), float(r[wi] or 0), r[0], r[1].strip()[:100]))
            except ValueError:
                pass
    ti = sum(l[0] for l in lines)
    tw = sum(l[1] for l in lines)
    print('total warp-inst %.2fM' % (ti / 1e6))
    for n, w, ln, src in sorted(lines, reverse=True)[:top]:
        print('%6.2f%% inst %5.1f%% stall  L%-4s %s' % (100 * n / ti, 100 * w / max(tw, 1), ln, src))


if __name__ == '__main__':
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40)
