// dts_loop_fast.cu -- the decision loop of dts_loop.cu compiled a second time,
// specialised to the mode every BASELINE config runs in (row-derived state,
// one shard, W = 0, DARTS+LUF): the other modes' branches and code are
// compiled out (see the mode predicates at the top of dts_loop.cu).  The host
// (dts_api.cu) launches dts_cta_kernel_fast when every instance of a launch
// is in that mode, dts_cta_kernel otherwise.
#define DTS_FAST 1
#include "dts_loop.cu"
