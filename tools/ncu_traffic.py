"""Write profiles/ncu_wa_traffic.json: DRAM bytes (read + write) per launch of the WA kernel
(k_wa_chunks: all nets in one launch) from one `ncu --set full` capture, for bench.py's
roofline.traffic.   python tools/ncu_traffic.py <report.ncu-rep>"""
import csv
import json
import subprocess
import sys


def dram_bytes(path, kname):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    ki = h.index('Kernel Name')
    for r in rows[2:]:
        if kname in r[ki]:
            b = 0.0
            for m in ('dram__bytes_read.sum', 'dram__bytes_write.sum'):
                i = h.index(m)
                scale = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}[u[i]]
                b += float(r[i].replace(',', '')) * scale
            return b
    return None


if __name__ == '__main__':
    b = dram_bytes(sys.argv[1], 'k_wa_chunks')
    out = {"dram_bytes_per_launch": b, "kernel": "k_wa_chunks", "source": [sys.argv[1]]}
    with open('profiles/ncu_wa_traffic.json', 'w') as f:
        json.dump(out, f, indent=1)
    print(out)
