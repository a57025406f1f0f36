// internal.h -- shared declarations of the Fringe-SGC library (not public).
#pragma once
#include <stdint.h>
#include <string>
#include <vector>
#include <array>
#include "../../include/fsgc.h"

// --------------------------------------------------------------- errors
void fsgc_set_error(const char* fmt, ...);

#define FSGC_FAIL(code, ...)            \
    do {                                \
        fsgc_set_error(__VA_ARGS__);    \
        return (code);                  \
    } while (0)

// triangle listing from the middle vertex (graph.cu builds the work units,
// count.cu runs them: support pass and triangle-core pass)
#define FSGC_SUP_CAPW 256        // max out(b) of a middle vertex with a warp table
#define FSGC_SUP_SEG 128         // in-neighbours per warp-table unit
#define FSGC_SUP_CHUNK 1024      // in-neighbours per block-table unit

// --------------------------------------------------------------- handles
struct fsgc_graph {
    uint64_t uid = 0;            // unique per loaded graph (plan cache key)
    int64_t n = 0, m = 0, max_degree = 0;
    int64_t* offsets = nullptr;  // [n+1]
    int32_t* adj = nullptr;      // [2m]
    int32_t* row = nullptr;      // [2m]
    int32_t* osrc = nullptr;     // [m]
    int32_t* odst = nullptr;     // [m]
    int32_t* order = nullptr;    // [n]
    int64_t* split = nullptr;    // [n]   CSR position of the first neighbour > v
    int64_t* oofs = nullptr;     // [n+1] oriented offsets: oriented index of
                                 //       CSR position p >= split[u] is
                                 //       oofs[u] + p - split[u]
    // Triangle listing from the MIDDLE vertex b (count.cu): every triangle
    // a < b < c is found from b, c in N+(a) & N+(b), a in N-(b).  Units =
    // (b, k), packed b << 32 | k, ordered by b:
    //   sup_units      1 <= out(b) <= sup_capw: the k-th FSGC_SUP_SEG slice of
    //                  N-(b), one warp with its own hash table of N+(b)
    //   sup_units_big  out(b) > sup_capw: the k-th FSGC_SUP_CHUNK slice of
    //                  N-(b), one block with a shared table of N+(b)
    uint64_t* sup_units = nullptr;   // [nsup_units]
    int64_t nsup_units = 0;
    uint64_t* sup_units_big = nullptr;   // [nsup_units_big]
    int64_t nsup_units_big = 0;
    int32_t sup_capw = FSGC_SUP_CAPW;    // out(b) split between the two (FSGC_SUP_CAPW knob)
    int64_t sup_maxout = 0;              // max out(b) of a block-table middle (table size)
    // rev[i - oofs[b]] = oriented index of (a, b) for the in-entry a = adj[i]
    // of row b (i in [offs[b], split[b])) -- the position of b in N+(a)
    int32_t* rev = nullptr;          // [m]
    int32_t sup_hash = 1;            // support pass: 1 listing kernels, 0 merge kernel
    // merge kernel (support_kernel) work list: every oriented edge (a, b)
    // sorted by merge length out(a) + out(b), with its endpoints (only for
    // graphs below FSGC_SUP_HASH_MIN_M edges or FSGC_SUP_MERGE_ONLY)
    int32_t* sorder = nullptr;   // [nsup_merge]
    int32_t* ssrc = nullptr;     // [nsup_merge]
    int32_t* sdst = nullptr;     // [nsup_merge]
    int64_t nsup_merge = 0;
    // hub bitmaps: vertices v >= hub_base (the highest-degree ones, ids are
    // degree ordered) have a dense n-bit adjacency bitmap (O(1) membership)
    int64_t hub_base = 0;        // == n when there are no hubs
    int64_t hub_words = 0;       // 32-bit words per bitmap
    uint32_t* hub_bits = nullptr;
    int device = 0;
};

struct fsgc_pattern {
    uint64_t uid = 0;                   // unique per compiled pattern (plan cache key)
    int n = 0;
    std::vector<std::array<int, 2>> edges;
    uint64_t adj[FSGC_MAX_PATTERN_VERTICES] = {};
    uint64_t core_mask = 0;
    std::vector<int> order;             // matching order (pattern vertex ids)
    std::vector<uint64_t> type_anchor;  // anchor set per fringe type
    std::vector<int> type_k;            // fringes per type
    uint64_t aut = 1, aut_core = 1, aut_core_labeled = 1, fringe_fact = 1;
};

// --------------------------------------------------------- device program
// Limits of one count pass (one core-isomorphism class of patterns).
#define FSGC_MAXC FSGC_MAX_CORE
#define FSGC_MAXQ FSGC_MAX_VENN_BITS
#define FSGC_MAXPROG 192
#define FSGC_MAXT 16
#define FSGC_MAXPATS FSGC_MAX_BATCH
#define FSGC_FC_STACK 64

enum { ROOT_ORIENTED = 0, ROOT_DIRECTED = 1, ROOT_VERTEX = 2 };

// A fringe program = one pattern's fringe types seen through one coset
// representative of the core's automorphisms (anchor sets as Venn bitsets).
struct FringeProg {
    uint8_t s;        // number of fringe types
    uint8_t pat;      // pattern index in the batch
    uint8_t depth;    // fc stack depth bound
    uint8_t ksum;     // total fringes (sum of k) -- for the 64-bit bound
    uint8_t anch[FSGC_MAXT];
    uint8_t k[FSGC_MAXT];
};

struct CoreProg {
    int32_t p;                  // core vertices
    int32_t q;                  // Venn bits (anchor positions)
    int32_t nprog;              // fringe programs
    int32_t npats;              // patterns in the pass
    int32_t root_mode;          // ROOT_*
    int32_t pad;
    uint8_t back[FSGC_MAXC];    // core-adjacency to earlier positions (bitmask)
    uint8_t gt[FSGC_MAXC];      // symmetry breaking: phi(i) > phi(j) for j in gt[i]
    int32_t mindeg[FSGC_MAXC];  // degree filter per position
    int8_t anchor_pos[FSGC_MAXQ];  // Venn bit -> core position
    int8_t pad2[2];
    FringeProg prog[FSGC_MAXPROG];
    // edge cores (p == 2): each program as (k tails on c0, l tails on c1,
    // m wedge fringes on {c0,c1}) for the Sec. 3.1 closed form
    uint8_t ek[FSGC_MAXPROG], el[FSGC_MAXPROG], em[FSGC_MAXPROG];
};

// fc of a program whose fringe types all have k = 1, by Moebius inversion on
// the partition lattice of its s types: fc = sum_pi coef(pi) prod_B Z[mask_B],
// Z[A] = sum of the Venn entries covering A; coef = prod (-1)^(|B|-1)(|B|-1)!
struct PartTerm {
    int32_t coef;
    uint8_t nb;                 // blocks
    uint8_t mask[7];            // Venn-bit anchor mask of each block
};

struct PassPlan {
    CoreProg prog;
    std::vector<std::vector<PartTerm>> terms;   // per program (empty: Listing 5)
    std::vector<int> members;          // indices into the caller's pattern array
    std::vector<uint64_t> divisor;     // per member: count = raw / divisor
    int root_pattern_vertex[FSGC_MAXPATS];
};

// pattern.cpp
int fsgc_core_isomorphism(const fsgc_pattern* ref, const fsgc_pattern* other, int* pos_of);
int fsgc_build_pass(const fsgc_pattern* const* pats, const std::vector<int>& members,
                    int no_symmetry_breaking, PassPlan* plan);
