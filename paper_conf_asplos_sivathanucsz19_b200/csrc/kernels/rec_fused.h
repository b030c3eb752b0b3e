// Host interface of the fused recurrent kernels (rec_fused.cu), LSTM family, bf16 path.
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>

#include "kernels.h"

namespace astra {

struct RecFwdArgs {
  int B, H, Hp, NG, T;      // T: total steps of the sequence (for hT / cT)
  int t0, t1;               // steps run by this launch
  int num_m, num_n;         // tiles: ceil(B/128) x NG/256
  int stages, nk, persistent;
  uint32_t idesc;           // instruction descriptor of the 128x256 bf16 MMA
  const float* WX;          // [T·B][NG] hoisted projection
  float* UH;                // [T·B][NG] recurrent projection (saved)
  float* C;                 // [(T+1)·B][Hp] cell state
  __nv_bfloat16* Hb;        // [(T+1)·B][Hp] h operand (TMA map A reads it)
  void* y;                  // optional output
  long ldy;
  int y_kind;               // 0 none, 1 bf16 external [T·B][ldy], 2 fp32 [T·B][ldy]
  float* hT;
  float* cT;
  GateParams gp;
  unsigned* flags;          // [num_m] row-block counters (zeroed before a persistent launch)
};

// mapA: Hb as a 3-D K-major map (inner Hp, rows B, z = T+1), box {64, 128};
// mapB: the U mirror [NG][Hp] K-major, box {64, 256}.
void lstm_rec_fwd_launch(int kind, const CUtensorMap& mapA, const CUtensorMap& mapB, RecFwdArgs a, cudaStream_t st);

}  // namespace astra
