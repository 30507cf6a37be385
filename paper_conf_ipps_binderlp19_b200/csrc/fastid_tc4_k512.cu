// fastid_tc4_k512.cu — the FastID tcgen05 kernel (fastid_tc4_impl.cuh) with 512-bit stages:
// 64-byte packed rows per TMA box (64B swizzle), 8-deep ring, 4 TMEM A stages (6 for the
// 32-wide query batch).  Measured best when the count matrices are written (FastID-1M).
#define FASTID_KBITS 512
#define FASTID_PRIMARY 1
#define FASTID_FN(name) name##_k512
#include "fastid_tc4_impl.cuh"
