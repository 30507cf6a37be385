// fastid_tc4_k1024.cu — the FastID tcgen05 kernel (fastid_tc4_impl.cuh) with 1024-bit
// stages: 128-byte packed rows per TMA box (128B swizzle: each database row is fetched in
// whole 128-byte lines, half as many stage hand-offs per tile), 4-deep ring of 16 KB
// stages, 2 TMEM A stages of 128 columns.  Measured 25-28 % faster than 512-bit stages on
// the few-query best-match searches (profiles/round2/sweep_kbits.txt).
#define FASTID_KBITS 1024
#define FASTID_NS 2
#define FASTID_NS32 2
#define FASTID_NP 4
#define FASTID_FN(name) name##_k1024
#include "fastid_tc4_impl.cuh"
