"""Write profiles/ncu_wa_traffic.json: DRAM bytes (read + write) per launch of the WA stage
(k_wa_chunks + k_wa_big) from one `ncu --set full` capture, for bench.py's roofline.traffic."""
import csv
import json
import subprocess
import sys


def dram_bytes(path, kname):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    ki = h.index('Kernel Name')
    tot = None
    for r in rows[2:]:
        if kname in r[ki]:
            b = 0.0
            for m in ('dram__bytes_read.sum', 'dram__bytes_write.sum'):
                i = h.index(m)
                scale = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}[u[i]]
                b += float(r[i].replace(',', '')) * scale
            tot = b
            break
    return tot


if __name__ == '__main__':
    chunks = dram_bytes(sys.argv[1], 'k_wa_chunks')
    big = dram_bytes(sys.argv[2] if len(sys.argv) > 2 else sys.argv[1], 'k_wa_big') or 0.0
    out = {"dram_bytes_per_launch": chunks + big, "k_wa_chunks": chunks, "k_wa_big": big,
           "source": sys.argv[1:]}
    json.dump(out, open('profiles/ncu_wa_traffic.json', 'w'), indent=1)
    print(out)
