/* up_kparams.h -- launch parameter block shared by the host (up_host.cpp) and
 * every generated kernel (embedded into NVRTC next to up_dev.cuh). */
#pragma once

#define UP_MAX_COLS 16

typedef struct {
    const unsigned int *col[UP_MAX_COLS];  /* limb planes of input column k (device) */
    long long ld[UP_MAX_COLS];             /* plane stride (elements), multiple of 4 */
    long long n;                           /* rows */
    unsigned int *out;                     /* eval: output planes */
    long long ld_out;
    unsigned long long *ws;                /* sum: 64-bit slot workspace (zeroed) */
    unsigned int *ticket;                  /* sum: last-block ticket (zeroed) */
    unsigned int *result;                  /* sum: LA-limb two's-complement partial */
    unsigned int *flags;                   /* sticky error flags (F_*) */
    unsigned int *scratch;                 /* per-thread global scratch (sin_P running sums) */
    long long scratch_stride;              /* elements between consecutive words of one thread */
    const int *group;                      /* group_aggregate: group id per row (NULL = one group) */
    unsigned long long *counts;            /* group_aggregate: rows per group */
} up_kparams;
