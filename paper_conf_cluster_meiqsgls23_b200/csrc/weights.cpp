// Parameter layout, deterministic init (R21) and the weights /
// optimizer-state files (SURVEY §8(b) "Weights file").
//
// Layout, per ANEE layer i (P141-P149 with readings R1, R5):
//   W_u[d][d_in]  W_e[d][d_e,in]  W_m[d][d]  a_s[d]  a_d[d]
// then the Graphormer layers (NEXT-3), the decoder (NEXT-2) when configured, and the head
// (P125, R12): W_1[d_h][d or k·d]  b_1[d_h]  w_2[d_h]  b_2[1].
#include <math.h>
#include <stdio.h>
#include <string.h>

#include <vector>

#include "occu_internal.h"

namespace occu {

ParamLayout make_layout(const occu_config &c) {
  ParamLayout L;
  size_t off = 0;
  for (int i = 0; i < c.L; ++i) {
    const int din = i == 0 ? c.F_n : c.d;
    const int dein = i == 0 ? c.F_e : c.d;
    L.d_in.push_back(din);
    L.de_in.push_back(dein);
    L.W_u.push_back(off); off += size_t(c.d) * din;
    L.W_e.push_back(off); off += size_t(c.d) * dein;
    L.W_m.push_back(off); off += size_t(c.d) * c.d;
    L.a_s.push_back(off); off += c.d;
    L.a_d.push_back(off); off += c.d;
  }
  L.head_in = c.d;
  const size_t d = size_t(c.d), dd = d * d;
  auto ffn = [&](FfnOff &f) {
    f.W1 = off; off += dd; f.b1 = off; off += d; f.W2 = off; off += dd; f.b2 = off; off += d;
  };
  for (int j = 0; j < c.graphormer; ++j) {     // Graphormer layers (NEXT-3), file order
    GphOff g;
    g.ln1_g = off; off += d; g.ln1_b = off; off += d;
    g.Wq = off; off += dd; g.bq = off; off += d;
    g.Wk = off; off += dd; g.bk = off; off += d;
    g.Wv = off; off += dd; g.bv = off; off += d;
    g.Wo = off; off += dd; g.bo = off; off += d;
    g.ln2_g = off; off += d; g.ln2_b = off; off += d;
    ffn(g.F);
    L.G.push_back(g);
  }
  if (c.readout == OCCU_READOUT_SET_DECODER) {
    L.dec = true;
    L.D.S = off; off += size_t(c.k) * d;
    ffn(L.D.P);
    for (MabOff *m : {&L.D.M1, &L.D.M2}) {
      m->Wq = off; off += dd; m->bq = off; off += d;
      m->Wk = off; off += dd; m->bk = off; off += d;
      m->Wv = off; off += dd; m->bv = off; off += d;
      m->Wo = off; off += dd; m->bo = off; off += d;
      m->ln1_g = off; off += d; m->ln1_b = off; off += d;
      ffn(m->F);
      m->ln2_g = off; off += d; m->ln2_b = off; off += d;
    }
    ffn(L.D.D);
    L.head_in = c.k * c.d;
  }
  L.W_1 = off; off += size_t(c.d_h) * L.head_in;
  L.b_1 = off; off += c.d_h;
  L.w_2 = off; off += c.d_h;
  L.b_2 = off; off += 1;
  L.total = off;
  return L;
}

// splitmix64 (counter form): output j (0-based) = mix(seed + (j+1)*golden).
static inline uint64_t splitmix64_at(uint64_t seed, uint64_t j) {
  uint64_t z = seed + (j + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

void init_flat(const occu_config &c, uint64_t seed, std::vector<float> &out) {
  const ParamLayout L = make_layout(c);
  out.assign(L.total, 0.f);
  struct T { size_t off, n; int fan_in; };
  std::vector<T> ts;
  for (int i = 0; i < c.L; ++i) {
    ts.push_back({L.W_u[i], size_t(c.d) * L.d_in[i], L.d_in[i]});
    ts.push_back({L.W_e[i], size_t(c.d) * L.de_in[i], L.de_in[i]});
    ts.push_back({L.W_m[i], size_t(c.d) * c.d, c.d});
    ts.push_back({L.a_s[i], size_t(c.d), 2 * c.d});
    ts.push_back({L.a_d[i], size_t(c.d), 2 * c.d});
  }
  // fan_in -1: constant 1 (LayerNorm gain), 0: constant 0 (LayerNorm bias)
  const size_t d = size_t(c.d), dd = d * d;
  auto ffn = [&](const FfnOff &f) {
    ts.push_back({f.W1, dd, c.d}); ts.push_back({f.b1, d, c.d});
    ts.push_back({f.W2, dd, c.d}); ts.push_back({f.b2, d, c.d});
  };
  for (const GphOff &g : L.G) {
    ts.push_back({g.ln1_g, d, -1}); ts.push_back({g.ln1_b, d, 0});
    for (size_t w : {g.Wq, g.Wk, g.Wv, g.Wo}) {
      ts.push_back({w, dd, c.d});
      ts.push_back({w + dd, d, c.d});            // its bias follows it
    }
    ts.push_back({g.ln2_g, d, -1}); ts.push_back({g.ln2_b, d, 0});
    ffn(g.F);
  }
  if (L.dec) {
    ts.push_back({L.D.S, size_t(c.k) * d, c.d});
    ffn(L.D.P);
    for (const MabOff *m : {&L.D.M1, &L.D.M2}) {
      for (size_t w : {m->Wq, m->Wk, m->Wv, m->Wo}) {
        ts.push_back({w, dd, c.d});
        ts.push_back({w + dd, d, c.d});          // its bias follows it
      }
      ts.push_back({m->ln1_g, d, -1}); ts.push_back({m->ln1_b, d, 0});
      ffn(m->F);
      ts.push_back({m->ln2_g, d, -1}); ts.push_back({m->ln2_b, d, 0});
    }
    ffn(L.D.D);
  }
  ts.push_back({L.W_1, size_t(c.d_h) * L.head_in, L.head_in});
  ts.push_back({L.b_1, size_t(c.d_h), L.head_in});
  ts.push_back({L.w_2, size_t(c.d_h), c.d_h});
  ts.push_back({L.b_2, 1, c.d_h});
  for (const T &t : ts) {
    if (t.fan_in <= 0) {
      for (size_t j = 0; j < t.n; ++j) out[t.off + j] = t.fan_in < 0 ? 1.f : 0.f;
      continue;
    }
    const double bound = 1.0 / sqrt(double(t.fan_in));
    for (size_t j = 0; j < t.n; ++j) {
      const uint64_t z = splitmix64_at(seed, t.off + j);
      const double u = double(z >> 11) * (1.0 / 9007199254740992.0);
      out[t.off + j] = float((2.0 * u - 1.0) * bound);
    }
  }
}

uint64_t fnv1a64(const void *data, size_t n) {
  const unsigned char *p = static_cast<const unsigned char *>(data);
  uint64_t h = 0xCBF29CE484222325ull;
  for (size_t i = 0; i < n; ++i) {
    h ^= p[i];
    h *= 0x100000001B3ull;
  }
  return h;
}

// File version: 1 = mean readout, 2 = decoder readout (+ u32 readout, k, heads), 3 = with
// Graphormer layers (+ u32 readout, k, heads, graphormer).
static uint32_t file_version(const occu_config &c) {
  return c.graphormer > 0 ? 3u : c.readout == OCCU_READOUT_SET_DECODER ? 2u : 1u;
}

// header: "OCCUW001", u32 version, L, F_n, F_e, d, d_h, aggr, msg, f32 slope
bool write_file(const char *path, const char magic[8], const occu_config &c,
                const std::vector<std::pair<const void *, size_t>> &chunks, std::string &err) {
  FILE *f = fopen(path, "wb");
  if (!f) {
    err = std::string("cannot open ") + path + " for writing";
    return false;
  }
  const uint32_t ver = file_version(c);
  const size_t next = ver == 3 ? 4 : ver == 2 ? 3 : 0;
  uint32_t hdr[8] = {ver, uint32_t(c.L), uint32_t(c.F_n), uint32_t(c.F_e), uint32_t(c.d),
                     uint32_t(c.d_h), uint32_t(c.aggr), uint32_t(c.msg)};
  const uint32_t ext[4] = {uint32_t(c.readout), uint32_t(c.k), uint32_t(c.heads), uint32_t(c.graphormer)};
  bool ok = fwrite(magic, 1, 8, f) == 8 && fwrite(hdr, 4, 8, f) == 8 &&
            fwrite(&c.slope, 4, 1, f) == 1 && fwrite(ext, 4, next, f) == next;
  uint64_t h = 0xCBF29CE484222325ull;
  for (auto &ch : chunks) {
    ok = ok && fwrite(ch.first, 1, ch.second, f) == ch.second;
    const unsigned char *p = static_cast<const unsigned char *>(ch.first);
    for (size_t i = 0; i < ch.second; ++i) {
      h ^= p[i];
      h *= 0x100000001B3ull;
    }
  }
  ok = ok && fwrite(&h, 8, 1, f) == 1;
  ok = (fclose(f) == 0) && ok;
  if (!ok) err = std::string("write failed: ") + path;
  return ok;
}

// Reads a file written by write_file; checks magic, config, size and checksum.
occu_status read_file(const char *path, const char magic[8], const occu_config &c,
                      std::vector<unsigned char> &payload, size_t expect_bytes, std::string &err) {
  FILE *f = fopen(path, "rb");
  if (!f) {
    err = std::string("cannot open ") + path;
    return OCCU_EINVAL;
  }
  std::vector<unsigned char> raw;
  unsigned char buf[1 << 16];
  size_t n;
  while ((n = fread(buf, 1, sizeof buf, f)) > 0) raw.insert(raw.end(), buf, buf + n);
  fclose(f);
  const uint32_t ver = file_version(c);
  const size_t next = ver == 3 ? 4 : ver == 2 ? 3 : 0;
  const size_t hdr = 8 + 32 + 4 + 4 * next;
  if (raw.size() < hdr + 8 || memcmp(raw.data(), magic, 8) != 0) {
    err = "bad magic or truncated file";
    return OCCU_EFORMAT;
  }
  uint32_t h[8], ext[4] = {0, 0, 0, 0};
  memcpy(h, raw.data() + 8, 32);
  float slope;
  memcpy(&slope, raw.data() + 40, 4);
  memcpy(ext, raw.data() + 44, 4 * next);
  if (h[0] != ver || int(h[1]) != c.L || int(h[2]) != c.F_n || int(h[3]) != c.F_e ||
      int(h[4]) != c.d || int(h[5]) != c.d_h || int(h[6]) != c.aggr || int(h[7]) != c.msg ||
      slope != c.slope ||
      (next >= 3 && (int(ext[0]) != c.readout || int(ext[1]) != c.k || int(ext[2]) != c.heads)) ||
      (next == 4 && int(ext[3]) != c.graphormer)) {
    err = "file config does not match the context config";
    return OCCU_EINVAL;
  }
  const size_t body = raw.size() - hdr - 8;
  if (body != expect_bytes) {
    err = "payload size mismatch";
    return OCCU_EFORMAT;
  }
  uint64_t sum;
  memcpy(&sum, raw.data() + hdr + body, 8);
  if (fnv1a64(raw.data() + hdr, body) != sum) {
    err = "checksum mismatch";
    return OCCU_EFORMAT;
  }
  payload.assign(raw.begin() + hdr, raw.begin() + hdr + body);
  return OCCU_OK;
}

}  // namespace occu
