// update_inst_0.cu -- explicit instantiations of the update and second-term kernels, D=1..8.
// (split across files so the 32 dimension variants compile in parallel)
#include "term.cuh"
#include "update_tc.cuh"
namespace egg {
#if !defined(EGG_DEV_D) || EGG_DEV_D == 1
template int run_update<1>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<1>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 2
template int run_update<2>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<2>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 3
template int run_update<3>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<3>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 4
template int run_update<4>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<4>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 5
template int run_update<5>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<5>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 6
template int run_update<6>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<6>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 7
template int run_update<7>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<7>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 8
template int run_update<8>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<8>(Workspace&, int64_t, int64_t);
#endif
}  // namespace egg
