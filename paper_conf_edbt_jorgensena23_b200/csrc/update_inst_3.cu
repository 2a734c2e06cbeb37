// update_inst_3.cu -- explicit instantiations of the update and second-term kernels, D=25..32.
// (split across files so the 32 dimension variants compile in parallel)
#include "term.cuh"
#include "update_tc.cuh"
namespace egg {
#if !defined(EGG_DEV_D) || EGG_DEV_D == 25
template int run_update<25>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<25>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 26
template int run_update<26>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<26>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 27
template int run_update<27>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<27>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 28
template int run_update<28>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<28>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 29
template int run_update<29>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<29>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 30
template int run_update<30>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<30>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 31
template int run_update<31>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<31>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 32
template int run_update<32>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<32>(Workspace&, int64_t, int64_t);
#endif
}  // namespace egg
