// update_inst_1.cu -- explicit instantiations of the update and second-term kernels, D=9..16.
// (split across files so the 32 dimension variants compile in parallel)
#include "term.cuh"
namespace egg {
template int run_update<9>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<9>(Workspace&, int64_t, int64_t);
template int run_update<10>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<10>(Workspace&, int64_t, int64_t);
template int run_update<11>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<11>(Workspace&, int64_t, int64_t);
template int run_update<12>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<12>(Workspace&, int64_t, int64_t);
template int run_update<13>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<13>(Workspace&, int64_t, int64_t);
template int run_update<14>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<14>(Workspace&, int64_t, int64_t);
template int run_update<15>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<15>(Workspace&, int64_t, int64_t);
template int run_update<16>(Workspace&, int64_t, int64_t, int32_t*);
template int run_second_term<16>(Workspace&, int64_t, int64_t);
}  // namespace egg
