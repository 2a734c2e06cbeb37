// update_inst_2.cu -- explicit instantiations of the update and second-term kernels, D=17..24.
// (split across files so the 32 dimension variants compile in parallel)
#include "term.cuh"
#include "update_tc.cuh"
namespace egg {
#if !defined(EGG_DEV_D) || EGG_DEV_D == 17
template int run_update<17>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<17>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 18
template int run_update<18>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<18>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 19
template int run_update<19>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<19>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 20
template int run_update<20>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<20>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 21
template int run_update<21>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<21>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 22
template int run_update<22>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<22>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 23
template int run_update<23>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<23>(Workspace&, int64_t, int64_t);
#endif
#if !defined(EGG_DEV_D) || EGG_DEV_D == 24
template int run_update<24>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<24>(Workspace&, int64_t, int64_t);
#endif
}  // namespace egg
