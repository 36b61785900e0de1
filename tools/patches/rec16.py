"""Apply the 16-byte density record variant (per-cell-size constant table; DESIGN.md §5.6 A/B)
to the tree in the current directory.  Used to build lib_ab/rec16.so for in-step A/B runs."""
p='paper_conf_dac_lindlrkp19_b200/csrc/dp_internal.h'
s=open(p).read()
s=s.replace('''// Per warp-group metadata of the WA chunk layout''','''struct CellType {
  double ox, oy;
  double wbd, hbd;
  float wb, hb, r;
  int flags;
};

// Per warp-group metadata of the WA chunk layout''')
s=s.replace('''  float4 *d_rec = nullptr;            // per slot: footprint box in tile-local bin units
  int2 *d_rec_rc = nullptr;           // per slot: (charge ratio r as float bits, i0 | j0 << 16)
  int32_t *d_rec_cell = nullptr;      // per slot: own cell index''','''  int4 *d_rec = nullptr;
  int32_t *d_cell_type = nullptr;
  float4 *d_type_f4 = nullptr;
  int32_t n_types = 0;''')
open(p,'w').write(s)
p='paper_conf_dac_lindlrkp19_b200/csrc/dp_api.cu'
s=open(p).read()
a=s.index('''  // sort records; padded by 8 so staged copies may round their range to 4-record multiples''')
b=s.index('''  // the maps of the hot path in one arena''')
s=s[:a]+'''  if ((st = dev_alloc(c, &c.d_rec, c.n_own + 8)) != DP_OK) return st;
  {
    std::map<std::pair<uint32_t, uint32_t>, int32_t> index;
    std::vector<int32_t> type(c.n_own);
    std::vector<float4> tf4;
    const double sq2 = 1.4142135623730951;
    for (int32_t i = 0; i < c.n_own; i++) {
      uint32_t kw, kh;
      std::memcpy(&kw, &w[i], 4);
      std::memcpy(&kh, &h[i], 4);
      auto it = index.find({kw, kh});
      if (it == index.end()) {
        const double wd = w[i], hd = h[i];
        const double ws = c.stretch ? std::max(wd, sq2 * c.bx) : wd;
        const double hs = c.stretch ? std::max(hd, sq2 * c.by) : hd;
        it = index.emplace(std::make_pair(kw, kh), (int32_t)tf4.size()).first;
        tf4.push_back(make_float4((float)(ws / c.bx), (float)(hs / c.by), (ws * hs > 0.0) ? (float)(wd * hd / (ws * hs)) : 0.f, 0.f));
      }
      type[i] = it->second;
    }
    if (tf4.size() > (size_t)(1 << 20)) return fail(DP_ERR_UNSUPPORTED, "more than 2^20 distinct cell sizes");
    if (tf4.empty()) tf4.push_back(make_float4(0.f, 0.f, 0.f, 0.f));
    c.n_types = (int32_t)tf4.size();
    if ((st = dev_upload(c, &c.d_cell_type, type)) != DP_OK) return st;
    if ((st = dev_upload(c, &c.d_type_f4, tf4)) != DP_OK) return st;
  }
'''+s[b:]
open(p,'w').write(s)
p='paper_conf_dac_lindlrkp19_b200/csrc/density.cu'
s=open(p).read()
s=s.replace('''  float4 *rec;
  int2 *rec_rc;   // (r as float bits, tile-local first bin i0 | j0 << 16)
  int *rec_cell;  // own cell index''','''  int4 *rec;
  const int *cell_type;
  const float4 *type_f4;''')
s=s.replace('''struct PlaceOut {
  float4 rec[kCountCells];
  int2 rc[kCountCells];
  int cell[kCountCells];
  int tile[kCountCells];
};''','''struct PlaceOut {
  int4 rec[kCountCells];
  int tile[kCountCells];
};''')
s=s.replace('''  float x[kCellsPerThread], y[kCellsPerThread], w[kCellsPerThread], h[kCellsPerThread];
  load_cells(a, i0, x, y, w, h);
  __syncthreads();
  float4 rec[kCellsPerThread];
  int rcy[kCellsPerThread], tl[kCellsPerThread], rank[kCellsPerThread];
  float rr[kCellsPerThread];''','''  float x[kCellsPerThread], y[kCellsPerThread], w[kCellsPerThread], h[kCellsPerThread];
  int ty[kCellsPerThread];
  load_cells(a, i0, x, y, w, h);
#pragma unroll
  for (int k = 0; k < kCellsPerThread; k++) {
    const int i = i0 + k * kCountThreads + threadIdx.x;
    ty[k] = i < a.n_own ? __ldg(a.cell_type + i) : 0;
  }
  __syncthreads();
  int4 rec[kCellsPerThread];
  int tl[kCellsPerThread], rank[kCellsPerThread];''')
s=s.replace('''    const int bi = f.bi, bj = f.bj;
    rec[k] = make_float4(fmaxf((float)(f.lx - bi), (float)-bi), fmaxf((float)(f.ly - bj), (float)-bj),
                         fminf((float)(f.hx - bi), (float)(a.mx - bi)), fminf((float)(f.hy - bj), (float)(a.my - bj)));
    rr[k] = __fdividef(w[k] * h[k], f.ws * f.hs);
    rcy[k] = (bi & mask) | ((bj & mask) << 16);''','''    rec[k] = make_int4(i, (f.bi & mask) | ((f.bj & mask) << 6) | (ty[k] << 12), __float_as_int((float)(f.lx - f.bi)),
                       __float_as_int((float)(f.ly - f.bj)));''')
s=s.replace('''    po.rec[slot] = rec[k];
    po.rc[slot] = make_int2(__float_as_int(rr[k]), rcy[k]);
    po.cell[slot] = i0 + k * kCountThreads + threadIdx.x;
    po.tile[slot] = tl[k];''','''    po.rec[slot] = rec[k];
    po.tile[slot] = tl[k];''')
s=s.replace('''    const int t = po.tile[j];
    const int pos = s_base[t] + (j - s_hist[t]);
    a.rec[pos] = po.rec[j];
    a.rec_rc[pos] = po.rc[j];
    a.rec_cell[pos] = po.cell[j];''','''    const int t = po.tile[j];
    a.rec[s_base[t] + (j - s_hist[t])] = po.rec[j];''')
s=s.replace('''struct RecBuf {
  float4 rec[kStageRecs + 8];
  int2 rc[kStageRecs + 8];
  int cell[kStageRecs + 8];
};''','''struct RecBuf {
  int4 rec[kStageRecs + 8];
};''')
s=s.replace('''  mbar_expect_tx(&st.bar[b], (unsigned)n * (with_cell ? 28u : 24u));
  if (n > 0) {
    RecBuf &B = st.buf[b];
    bulk_g2s(B.rec, a.rec + b0, 16u * n, &st.bar[b]);
    bulk_g2s(B.rc, a.rec_rc + b0, 8u * n, &st.bar[b]);
    if (with_cell) bulk_g2s(B.cell, a.rec_cell + b0, 4u * n, &st.bar[b]);
  }''','''  (void)with_cell;
  mbar_expect_tx(&st.bar[b], (unsigned)n * 16u);
  if (n > 0) bulk_g2s(st.buf[b].rec, a.rec + b0, 16u * n, &st.bar[b]);''')
s=s.replace('''__device__ __forceinline__ void rec_overlaps(const float4 q, float ox3[3], float oy3[3]) {
#pragma unroll
  for (int d = 0; d < 3; d++) {
    ox3[d] = fmaxf(fminf(q.z, (float)(d + 1)) - fmaxf(q.x, (float)d), 0.f);
    oy3[d] = fmaxf(fminf(q.w, (float)(d + 1)) - fmaxf(q.y, (float)d), 0.f);
  }
}''','''__device__ __forceinline__ float rec_overlaps(const DenArgs &a, const int4 q, float ox3[3], float oy3[3]) {
  const float4 T = __ldg(a.type_f4 + ((unsigned)q.y >> 12));
  const float fx = __int_as_float(q.z), fy = __int_as_float(q.w);
  const float hx = fx + T.x, hy = fy + T.y;
#pragma unroll
  for (int d = 0; d < 3; d++) {
    ox3[d] = fmaxf(fminf(hx, (float)(d + 1)) - fmaxf(fx, (float)d), 0.f);
    oy3[d] = fmaxf(fminf(hy, (float)(d + 1)) - fmaxf(fy, (float)d), 0.f);
  }
  return T.z;
}''')
s=s.replace('''      const float4 q = B.rec[cc.off + k];
      const int2 rc = B.rc[cc.off + k];
      const float r = __int_as_float(rc.x) * scale_fx;   // r 2^29
      const int i0 = rc.y & 0xffff, j0 = rc.y >> 16;
      float ox3[3], oy3[3];
      rec_overlaps(q, ox3, oy3);''','''      const int4 q = B.rec[cc.off + k];
      float ox3[3], oy3[3];
      const float r = rec_overlaps(a, q, ox3, oy3) * scale_fx;
      const int i0 = q.y & 63, j0 = (q.y >> 6) & 63;''')
s=s.replace('''          if (old + u < old)   // wrapped: 2^32 units (8 bin areas) go straight to the map''','''          if (old + u < old && ox + i0 + di < (size_t)a.mx && oy + j0 + dj < (size_t)a.my)''')
s=s.replace('''      const float4 q = B.rec[cc.off + k];
      const int2 rc = B.rc[cc.off + k];
      const float r = __int_as_float(rc.x);
      const int i0 = rc.y & 0xffff, j0 = rc.y >> 16;
      float ox3[3], oy3[3];
      rec_overlaps(q, ox3, oy3);''','''      const int4 q = B.rec[cc.off + k];
      float ox3[3], oy3[3];
      const float r = rec_overlaps(a, q, ox3, oy3);
      const int i0 = q.y & 63, j0 = (q.y >> 6) & 63;''')
s=s.replace('''        const int gc = a.cell_begin + B.cell[cc.off + k];''','''        const int gc = a.cell_begin + q.x;''')
s=s.replace('''        a.force[B.cell[cc.off + k]] = make_float2(-area * r * fx, -area * r * fy);''','''        a.force[q.x] = make_float2(-area * r * fx, -area * r * fy);''')
s=s.replace('''  a.rec = c.d_rec;
  a.rec_rc = c.d_rec_rc;
  a.rec_cell = c.d_rec_cell;''','''  a.rec = c.d_rec;
  a.cell_type = c.d_cell_type;
  a.type_f4 = c.d_type_f4;''')
open(p,'w').write(s)
print("rec16 patch applied")
