// update_inst_1.cu -- explicit instantiations of the update and second-term kernels, D=9..16.
// (split across files so the 32 dimension variants compile in parallel)
#include "term.cuh"
#include "update_tc.cuh"
namespace egg {
#if !defined(EGG_DEV_D) || EGG_DEV_D == 9
template int run_update<9>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<9>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 10
template int run_update<10>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<10>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 11
template int run_update<11>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<11>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 12
template int run_update<12>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<12>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 13
template int run_update<13>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<13>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 14
template int run_update<14>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<14>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 15
template int run_update<15>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<15>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 16
template int run_update<16>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<16>(Workspace&, int64_t, int64_t);
#endif
}  // namespace egg
