// variant_inst.h -- expands GTR_VARIANT_INSTANCES into GTR_INST(M, P, F, NT, FLAGS)
// lines for the variant(s) this translation unit builds (see build.py).
#pragma once
#if defined(GTR_V_MODE)
#ifndef GTR_V_FLAGS
#define GTR_V_FLAGS 0
#endif
#define GTR_VARIANT_INSTANCES GTR_INST(GTR_V_MODE, GTR_V_PL, GTR_V_FOLD, GTR_V_NT, GTR_V_FLAGS)
#elif defined(GTR_V_GROUP_NT)
#ifndef GTR_V_FLAGS
#define GTR_V_FLAGS 0
#endif
#define GTR_GROUP_PL(M, P)                                                    \
    GTR_INST(M, P, true, GTR_V_GROUP_NT, GTR_V_FLAGS)                         \
    GTR_INST(M, P, false, GTR_V_GROUP_NT, GTR_V_FLAGS)
#define GTR_GROUP_M(M)                                                        \
    GTR_GROUP_PL(M, gtr::PL_RUNTIME) GTR_GROUP_PL(M, gtr::PL_GLOBAL)           \
    GTR_GROUP_PL(M, gtr::PL_SHARED_STATIC) GTR_GROUP_PL(M, gtr::PL_STACK)  \
    GTR_GROUP_PL(M, gtr::PL_COALESCED)
#if defined(GTR_V_SPMD_ONLY)
#define GTR_VARIANT_INSTANCES GTR_GROUP_M(gtr::SPMD)
#else
#define GTR_VARIANT_INSTANCES GTR_GROUP_M(gtr::CSM) GTR_GROUP_M(gtr::SPMD)
#endif
#else
#error "variant TU needs GTR_V_MODE.. or GTR_V_GROUP_NT"
#endif
