// tt_check.cuh -- device-side bounds checks of the checked build.
//
// `python paper_conf_sc_goldfarbjk13_b200/build.py --checked` compiles every
// kernel with -DTT_CHECKED into libtt_checked.so (separate objects); a failed
// check prints the condition and traps, so the launch fails with a CUDA error
// the caller sees.  The product build compiles the checks away.  Used where
// compute-sanitizer cannot run.
#pragma once
#ifdef TT_CHECKED
#include <cstdio>
#define TT_DCHECK(c)                                                                           \
    do {                                                                                       \
        if (!(c)) {                                                                            \
            printf("TT_DCHECK failed %s:%d block %d thread %d: %s\n", __FILE__, __LINE__,       \
                   (int)blockIdx.x, (int)threadIdx.x, #c);                                     \
            __trap();                                                                          \
        }                                                                                      \
    } while (0)
#else
#define TT_DCHECK(c) \
    do {             \
    } while (0)
#endif
