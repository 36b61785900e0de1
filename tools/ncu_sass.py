"""Per-opcode instruction / stall breakdown and hottest SASS lines of one kernel in an .ncu-rep."""
import collections
import csv
import re
import subprocess
import sys


def main(path, kregex, top=25):
    out = subprocess.run(['ncu', '-i', path, '--page', 'source', '--csv', '-k', f'regex:{kregex}', '--launch-count', '1',
                          '--print-source', 'sass'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hi = [i for i, r in enumerate(rows) if 'Source' in r and 'Instructions Executed' in r][0]
    h = rows[hi]
    si, ii, wi = h.index('Source'), h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
    ops, st = collections.Counter(), collections.Counter()
    lines = []
    for r in rows[hi + 1:]:
        try:
            n, w = float(r[ii] or 0), float(r[wi] or 0)
        except (ValueError, IndexError):
            continue
        src = r[si].strip()
        op = re.sub(r'^@!?U?P\w+\s+', '', src).split(' ')[0]
        ops[op] += n
        st[op] += w
        lines.append((w, n, src))
    tot, tws = sum(ops.values()), sum(st.values())
    print('total warp-inst %.2fM, stall samples %d' % (tot / 1e6, tws))
    for op, n in ops.most_common(top):
        print('%-22s %6.2f%% inst  %5.1f%% stall' % (op, 100 * n / tot, 100 * st[op] / max(tws, 1)))
    print('--- hottest lines by stall samples')
    for w, n, src in sorted(lines, reverse=True)[:15]:
        print('%5.1f%% stall %6.2f%% inst  %s' % (100 * w / max(tws, 1), 100 * n / tot, src[:90]))


if __name__ == '__main__':
    main(sys.argv[1], sys.argv[2])
