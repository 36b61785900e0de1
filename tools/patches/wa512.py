"""A/B variant: WA CTAs of 512 threads (16 warps, one CTA per SM, <= 88 registers) so a density
walker CTA fits on the same SM (shared memory 101 + 92 KB, registers 45K + 20K)."""
import sys
nreg = int(sys.argv[1]) if len(sys.argv) > 1 else 88
p='paper_conf_dac_lindlrkp19_b200/csrc/dp_internal.h'
s=open(p).read()
s=s.replace('constexpr int kWaThreads = 256;','constexpr int kWaThreads = 512;')
s=s.replace('constexpr int kBigThreads = 256;','constexpr int kBigThreads = 512;')
s=s.replace('constexpr int kWarpNetThreads = 256;','constexpr int kWarpNetThreads = 512;')
open(p,'w').write(s)
p='paper_conf_dac_lindlrkp19_b200/csrc/wa.cu'
s=open(p).read()
s=s.replace('__global__ void __launch_bounds__(kWaThreads, 2) k_wa_chunks(const WaArgs a0) {',
            '__global__ void __maxnreg__(%d) k_wa_chunks(const WaArgs a0) {' % nreg)
open(p,'w').write(s)
print("wa512 patch applied", nreg)
