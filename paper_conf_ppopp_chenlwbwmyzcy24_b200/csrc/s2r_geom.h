// s2r_geom.h — compile-time geometry of the TC_S2R kernels, shared by the planner (host) and
// the kernels (device) so both agree on tile sizes and the stencil2row smem pitch.
#pragma once

namespace csx {

// Smallest pitch >= min_pitch (doubles) with pitch mod 16 in {4, 12}: the two 4x4 FP64
// requests of an m8n8k4 A fragment then hit 16 distinct 8-byte bank pairs for any column
// (P.1736-1757, Fig 5: 266 -> 268).  planner.cpp's fragment_conflicts() model proves it.
constexpr int s2r_pitch(int min_pitch) {
  int p = min_pitch;
  while (p % 16 != 4 && p % 16 != 12) ++p;
  return p;
}

template <int NK, bool PAD = true>
struct S2R2D {
  static constexpr int NKV = NK;
  static constexpr int SW = NK + 1;            // strip width: outputs per strip row
  static constexpr int KS = (NK * NK + 3) / 4; // k-slices per weight matrix (K = nk^2 -> 4*KS)
  static constexpr int BM = 32;                // CTA output rows   (Table 4: 32 x 64 for nk=7)
  static constexpr int BN = 8 * SW;            // CTA output cols = one warp-wide tessellation
  static constexpr int RR = BM + NK - 1;       // input region rows
  static constexpr int RC = BN + NK - 1;       // input region cols
  static constexpr int NE = RR * RC;           // LUT entries
  static constexpr int STRIPS = 8;             // stencil2row rows per CTA (+1 dirty row)
  static constexpr int PITCH = PAD ? s2r_pitch(NK * RR) : NK * RR;
  static constexpr int R = (NK - 1) / 2;
  // B200 staging: the raw input region arrives by cp.async.bulk rows (16-B aligned, hence the
  // ODD shift) in a 2-stage ring filled by one producer warp; 8 consumer warps scatter it
  // through the LUT into A/B and run the dual tessellations (4 output rows each).
  static constexpr int ODD = R & 1;
  static constexpr int TPR = (ODD + RC + 1) / 2 * 2;  // raw staged row length (even)
  static constexpr int RAW = RR * TPR;                 // doubles per raw stage
  // A/B are double-buffered (tile k+1 is scattered while slower warps still run tile k's
  // tessellation: one CTA barrier per tile).  nk = 7 keeps one raw stage (refilled during the
  // tessellation) so that two CTAs fit an SM; smaller windows keep two (measured).
  static constexpr int RAW_STAGES = NK >= 7 ? 1 : 2;
  static constexpr int AB_BUFS = 2;
  static constexpr int AB = 2 * (STRIPS + 1) * PITCH;  // doubles per A/B buffer
  static constexpr int NCW = 8;                        // consumer warps
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int SMEM = AB_BUFS * AB * 8 + NE * 4 + RAW_STAGES * RAW * 8;
};

template <int NK>
struct S2R1D {
  static constexpr int SW = NK + 1;
  static constexpr int NF = (SW + 7) / 8;      // N fragments (reading A7)
  static constexpr int KS = (NK + 3) / 4;
  static constexpr int NDT = 16;               // dual tessellations per CTA tile
  static constexpr int BN = 8 * SW * NDT;
  static constexpr int RC = BN + NK - 1;
  static constexpr int NE = RC;
  static constexpr int STRIPS = BN / SW;       // = 128
  static constexpr int PITCH = s2r_pitch(4 * KS);
  static constexpr int R = (NK - 1) / 2;
  static constexpr int NT = 128;
  static constexpr int SMEM = 2 * (STRIPS + 1) * PITCH * 8 + NE * 8;
};

#ifndef S2R3D_BM
#define S2R3D_BM 16  // round 2: 16 (4 rows per warp); round 1 / Table 4's 8 x 64 block: 8
#endif
template <int NK>
struct S2R3D {
  static constexpr int SW = NK + 1;
  static constexpr int KS = (NK * NK + 3) / 4;
  static constexpr int BM = S2R3D_BM;         // rows per CTA tile (4 warps x BM / 4 rows)
  static constexpr int BN = 8 * SW;
  static constexpr int RR = BM + NK - 1;
  static constexpr int RC = BN + NK - 1;
  static constexpr int NE = RR * RC;
  static constexpr int STRIPS = 8;
  static constexpr int PITCH = s2r_pitch(NK * RR);
  static constexpr int R = (NK - 1) / 2;
  static constexpr int NT = 128;               // 4 warps x BM / 4 output rows
  static constexpr int ZCHUNK = 64;            // output planes per work item
  static constexpr int SMEM = 2 * (STRIPS + 1) * PITCH * 8 + NE * 8 + RR * RC * 8;
};

}  // namespace csx
