// kernels.cuh -- argument blocks of the per-level sm_100a kernels (train.cu).
#pragma once
#include "common.cuh"

namespace gbdt {

// Node table of one level: node j (ascending heap id) with its totals ("G ... the total
// gradients of the node to split").
struct NodeTab {
  int32_t* K;       // [1] active nodes
  int32_t* heap;    // [Kcap] heap ids
  double* G;        // [Kcap]
  double* H;        // [Kcap]
  int32_t* cnt;     // [Kcap]
  double* pterm;    // [Kcap] G^2/(H+lambda), the parent term of Eq. 2
};

// Fenwick-tree look-back storage: top block of every tile (see split_find in train.cu).
struct Fenwick {
  double* G;
  double* H;
  int32_t* C;
  int32_t* F;   // 1: the block contains a segment head
  int32_t* E;   // publication flag = level epoch
};

struct TileArgs {
  const float* val;
  const int32_t* ins;
  Tables tb;
  int m;
  int a_base;          // global id of local attribute 0
  const int32_t* Kp;   // active nodes at this level
  int* counter;        // dynamic tile claim counter (reset per level)
};

struct SplitArgs {
  TileArgs t;
  const double2* gh;
  NodeTab nodes;
  const double* segPG;   // [m*K] present totals per segment (only with missing values)
  const double* segPH;
  double lam;
  const int32_t* epochp;
  Fenwick fw;
  Rec* rec;              // per-piece records (appended)
  int* nrec;
  unsigned long long* gkey;  // [Kcap] per node max gain key
  int shard;
  int totals_only;       // 1: write segPG/segPH instead of evaluating gains
  double* segPG_out;
  double* segPH_out;
};

struct PartArgs {
  TileArgs t;
  const uint8_t* side;    // per instance: 0 drop, 1 high, 2 low
  uint32_t* tile_cnt;     // [T] packed hi | lo<<16
  int32_t* segH;          // [m*K]
  int32_t* segL;
  const unsigned long long* tile_pre;  // [T] packed hi | lo<<32 exclusive
  const unsigned long long* seg_pre;   // [m*K]
  const int64_t* out_hi;  // [m*K]
  const int64_t* out_lo;
  float* val_out;
  int32_t* ins_out;
};

}  // namespace gbdt
