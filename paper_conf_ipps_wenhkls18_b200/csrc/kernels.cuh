// kernels.cuh -- argument blocks of the per-level sm_100a kernels (train.cu, levels.cu).
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

struct TileArgs {
  const float* val;
  const int32_t* ins;
  Tables tb;
  int m;
  int a_base;          // global id of local attribute 0
  const int32_t* Kp;   // active nodes at this level
  int* counter;        // dynamic tile claim counter (reset per level)
  const uint8_t* sflag = nullptr;  // [m] 1: attribute on the short path (k_short_*); nullptr: none
};

// Attributes whose whole root list has at most 32 entries (the typical sparse attribute)
// take the short path at levels 0-5 (K <= 32): a lane per list entry, 32/W lists per warp
// (levels.cu k_short_split / _count / _scatter).
struct ShortList {
  const int32_t* attrs = nullptr;  // shard-local ids, longest root list first
  int n = 0;
  const int2* batch = nullptr;     // warp batches: (first index into attrs, count | log2 W << 16)
  int nb = 0;
  const uint8_t* jl = nullptr;     // per list entry: its node j at this level (nullptr: root, j = 0)
  uint8_t* jl_out = nullptr;       // the next level's, written by the scatter (nullptr: not needed)
  // In-place mode (trees of depth <= 6): the short lists are never partitioned.  They stay in the
  // root layout (cs0 / cl0, the root values, g in gsh / hsh at root positions), every entry keeps
  // its node index in jl (0xff: its node became a leaf), updated in place by k_short_update, and
  // the split find sorts a list's lanes by node (stable: the partitioned order) before its scans.
  int inplace = 0;
  const int64_t* cs0 = nullptr;
  const int64_t* cl0 = nullptr;
  const float* val0 = nullptr;
  const int32_t* ins0 = nullptr;
  double* gsh = nullptr;
  double* hsh = nullptr;
};



// Per-chunk descriptor written by k_chunk_agg for the split-find kernels (32 bytes).
struct ChunkDesc {
  long long p0;   // first entry
  long long se;   // end of the segment holding the chunk's first entry
  int len;        // entries
  int a;          // attribute (shard-local)
  int jf;         // bits 0-15: segment (node) j of the first entry; 16: the chunk starts at that
                  // segment's start; 17: the chunk lies in that one segment; 18: vnext valid
  float vnext;    // value of the entry after the chunk when it is in the same attribute (plain)
};
constexpr int kDescHead0 = 1 << 16, kDescSingle = 1 << 17, kDescNext = 1 << 18;

struct SplitArgs {
  TileArgs t;
  ChunkDesc* desc;       // [C]
  int32_t* genlist;      // [C] chunks that cross a segment boundary (k_sf_gen), appended
  int32_t* ngen;
  int rle;               // the level's values live in runs (t.val is not maintained)
  const double* g;       // per instance
  const double* h;       // per instance (mode 2)
  double* glist;         // per list entry: g of the entry's instance (written by k_tile_agg)
  double* hlist;         // per list entry: h (mode 2)
  unsigned long long* cagg;   // [C][5] chunk aggregate: fixed-point g, h (lo,hi each), count | flags
  unsigned long long* carry;  // [C][5] exclusive segmented prefix of the chunk (same layout)
  unsigned long long* sgrp;   // scan scratch (group aggregates / carries)
  NodeTab nodes;
  const double* segPG;   // [m*K] present totals per segment (only with missing values)
  const double* segPH;
  double lam;
  const int32_t* epochp;
  const int32_t* fx;     // [2] fixed-point scales F_g, F_h of this tree (value * 2^F fits in 2^125)
  Rec* rec;              // node-best records (appended)
  int* nrec;
  unsigned long long* gkey;  // [Kcap] per node max gain key
  int shard;
  double* segPG_out;     // present totals per segment (missing values), written by k_chunk_agg
  double* segPH_out;     //   + k_seg_totals
  int32_t* segEnd;       // [m*K] chunk holding the segment's last entry if the segment began in an
                         // earlier chunk, else -1; nullptr: no missing values
  // the attributes not on the short path (k_seg_totals walks only their segments while the short
  // path is active); nullptr: every attribute
  const int32_t* longa = nullptr;
  int nlong = 0;
};

struct PartArgs {
  TileArgs t;
  const double* g_in;     // g-list (h-list) of this level, moved with the entries
  const double* h_in;
  double* g_out;
  double* h_out;
  const int32_t* epochp;
  const uint8_t* side;    // per instance: 0 drop, 1 high, 2 low
  const uint32_t* hbit;   // per instance: bit = [side == 1] (dense count, chunks inside one segment)
  const int32_t* cidx;    // [K] next-level index of node j's high child, -1 if j became a leaf
  uint8_t* slist;         // per list entry: side of its instance (k_part_count -> k_part_scatter)
  int32_t* segH;          // [m*K] counted (missing values) or derived from node counts (dense)
  int32_t* segL;
  unsigned long long* ccnt;  // [C][2] chunk (high | low << 32) counts, reset flag
  unsigned long long* cpre;  // [C][2] exclusive count of the attribute before the chunk
  unsigned long long* sgrp;  // scan scratch
  const unsigned long long* seg_pre;   // [m*K] exclusive count of the attribute before the segment
  const int64_t* out_hi;  // [m*K]
  const int64_t* out_lo;
  float* val_out;
  int32_t* ins_out;
  // Next level's chunk aggregates, accumulated by the scatter (no missing values): exact
  // fixed-point (g, h) per chunk (words 0-3 of each 5-word record; k_desc writes word 4)
  unsigned long long* cagg_next;  // nullptr: the next level runs k_chunk_agg instead
  Tables nxt;                     // next level's tables (from the plan)
  const int32_t* fx;              // [2] fixed-point scales of this tree
};

struct PlanArgs {
  int m;
  int counted;            // 1: segH/segL were counted (missing values); 0: derive from node counts
  const int32_t* Kp;      // current K
  const int32_t* Knp;     // next K
  const int32_t* cidx;
  const int32_t* ncnt;    // next-level node counts
  int32_t* segH;
  int32_t* segL;
  unsigned long long* seg_pre;
  int64_t* out_hi;
  int64_t* out_lo;
  int64_t* len_tmp;       // [m]
  unsigned long long* el; // [m+1][2] scan elements: padded list length | chunks << 32
  unsigned long long* egrp;
  unsigned egroups;
  const int32_t* mp1;     // m + 1 (device)
  Tables nxt;
  const uint8_t* sflag = nullptr;  // short-path attributes: left out of nxt.lc when K' <= 32
  int inplace = 0;                 // in-place short lists: their child lists are empty, no segments
};

struct RunArgs {
  int m;
  const int32_t* Kp;
  const int32_t* Knp;
  const int32_t* cidx;
  Tables cur, nxt;                 // run tables of this level / the next (nxt.seg_start from the plan)
  const uint8_t* slist;
  const unsigned long long* cpre;  // [C][2] the partition's chunk prefix counts (attribute-relative)
  int32_t* run_seg;                // [Rcap] parent segment of each run
  unsigned long long* run_hl;      // [Rcap] h_r | l_r << 32
  unsigned long long* cnt;         // [Rcap][2] scan elements (h_r | l_r << 32, segment head)
  unsigned long long* fl;          // [Rcap+1][2] scan elements ([h_r>0] | [l_r>0] << 32, 0)
  int32_t* Rp1;                    // R + 1 (length of the flag scan)
  unsigned long long* sgrp;        // scan scratch
  unsigned groups;
};

// fused.cu: dense levels below the root, partition of level l + split find of level l+1 in one
// pass (no missing values, g-list only, K <= kFusedMaxK nodes per level, i.e. max_depth <= 8)
constexpr int kFusedMaxK = 64;
struct FusedPlan {            // device, written by k_fused_plan
  long long n_act;            // entries per attribute list at level l (instances in active nodes)
  long long stride;           // padded list length at level l (attribute a starts at a * stride)
  long long n_next, stride_next;
  int tpa;                    // 2048-entry tiles per attribute
  int T;                      // tiles of the level (0: no child to scan)
  int K, Kn;                  // nodes at level l, l+1
  int epoch;                  // the level epoch of the records / look-back status words
  int off[kFusedMaxK + 1];    // segment start of node j within an attribute list, off[K] = n_act
  int cidx[kFusedMaxK];       // high child of node j at level l+1 (low = +1), -1: became a leaf
  int offn[2 * kFusedMaxK + 1];  // child segment starts in the next level's lists
  int pj[2 * kFusedMaxK];     // parent of child c
};
// Per child side (0 high, 1 low) of a tile's last segment piece: entries, exact fixed-point
// (g, h) sums, value and level position of the last one (fused.cu tile records / carries)
struct __align__(16) TSide {
  unsigned long long g_lo, g_hi, h_lo, h_hi;
  long long pos;
  int cnt;
  float val;
};
struct __align__(16) TRec {
  TSide s[2];
};
struct FusedArgs {
  const float* val;           // level l lists (val, ins, g-list)
  const int32_t* ins;
  const double* gl;
  float* val_out;             // level l+1 lists (when the children are partitioned again)
  int32_t* ins_out;
  double* g_out;
  const uint32_t* hbit;       // instance -> high-child bit of level l's splits
  const FusedPlan* plan;
  NodeTab nxt;                // the children: G, H, pterm
  // per tile (fused_carve): records, scanned carries, side bits
  TRec* tagg;
  TRec* tinc;
  TRec* tgagg;
  TRec* tgcarry;
  unsigned char* treset;
  unsigned char* tseen;
  unsigned char* tgf;
  unsigned char* tbits;       // [tiles][256]: bit k of byte i = entry 8 i + k goes high
  Rec* cta_rec;               // [CTAs][2 kFusedMaxK] node-best records of each k_fused CTA
  int warp_tiles;             // 1: single-piece tiles go to k_fusedw (0: every tile to k_fused; A/B)
  int* mcount;                // tiles holding several segment pieces (k_tile_agg appends them)
  int* mlist;
  const int32_t* fx;          // [2] fixed-point scales of this tree
  double lam;
  int m, a_base, shard;
  Rec* rec;                   // node-best records of level l+1 (appended)
  int* nrec;
  unsigned long long* gkey;
};
size_t fused_tile_bytes(int64_t max_tiles);
int64_t fused_tiles(int64_t n, int m);
void fused_carve(FusedArgs& A, void* base, int64_t max_tiles);
void fused_init(int sms);
unsigned fused_grid(int hmode);
void fused_plan(FusedPlan* P, const NodeTab& cur, const NodeTab& nxt, const int32_t* cidx, const int* epoch, int m,
                unsigned long long* lent, int lvl, int* mcount, cudaStream_t st);
void fused_pass(const FusedArgs& A, int hmode, bool write, int64_t max_tiles, cudaStream_t st);
void fused_mark(const FusedPlan* P, const int32_t* Kp, const int32_t* cidx, const Rec* winner, int shard, int a_base,
                const int32_t* ins, const uint32_t* hbit, uint32_t* bits, int64_t n, int Kl, int sms, cudaStream_t st);

// levels.cu launchers
struct LevelKernels {
  int sms = 148;
  unsigned grid_fast[3][2] = {{0}};  // [hmode][rle]
  unsigned grid_gen = 0;
  unsigned grid_short = 0;
  unsigned grid_sl = 0;  // k_short_split
  unsigned grid_agg[3] = {0};
  unsigned grid_fused = 0;
  unsigned grid_scatter[3][2] = {{0}}, grid_count = 0, grid_count_dense = 0, grid_agg_list[3] = {0};  // scatter: [hmode][agg]
  void init(int device);
  // a3/a4: tile aggregates (+ g/h lists) and the exact segmented carry scan
  static unsigned scan_groups(int64_t max_chunks);
  void tile_prefix(const SplitArgs& A, int hmode, bool gather, unsigned groups, cudaStream_t st);
  void split_find(const SplitArgs& A, int hmode, bool missing, bool rle, cudaStream_t st);
  void seg_totals(const SplitArgs& A, int hmode, cudaStream_t st);
  // a8: count -> exact scan -> plan (next level's tables), then the stable scatter
  void partition_count(const PartArgs& A, const PlanArgs& P, bool counted, unsigned groups, cudaStream_t st,
                       const ShortList* sl = nullptr);
  void partition_scatter(const PartArgs& A, int hmode, const RunArgs* rle, cudaStream_t st,
                         const ShortList* sl = nullptr);
  // split find of the short-path attributes (root: gathers their g-lists too)
  void short_split(const SplitArgs& A, const ShortList& S, int hmode, bool gather, cudaStream_t st);
  // a3: the level's chunk descriptors and scan flags when the previous scatter accumulated the
  // chunk aggregates, then the exact carry scan
  void chunk_desc(const SplitArgs& A, unsigned groups, cudaStream_t st);
  // a4-a6 with RLE and no missing values: run totals from the level's g-list, then the
  // split find over the runs (racc: [Rcap][5] exact fixed-point g, h per run as scan records,
  // rcar: their exclusive segmented prefixes, rsg: scan scratch of 5 * groups + 8 words)
  void run_split(const SplitArgs& A, int hmode, bool root, unsigned long long* racc, unsigned long long* rcar,
                 unsigned long long* rsg, unsigned groups, cudaStream_t st);
  // RLE split ablation (Fig. 6): decompress a level's runs into its value list; compress
  // the next level's value list (per node segment) into its run tables
  void rle_decompress(const Tables& tb, float* val, cudaStream_t st);
  void rle_encode(const Tables& tn, int m, const int32_t* Knp, const float* val, uint32_t* cnt, uint32_t* sbits,
                  size_t sbits_bytes, cudaStream_t st);
};

}  // namespace gbdt
