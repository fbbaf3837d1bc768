#include "nccl_dyn.h"

#include <dlfcn.h>

#include <mutex>

namespace ooo {

namespace {
NcclApi g_api;
const char *g_why = "not loaded";
std::once_flag g_once;

void load() {
  void *h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  if (!h) {
    g_why = "dlopen(libnccl.so.2) failed";
    return;
  }
#define OOO_SYM(field, name)                                           \
  g_api.field = reinterpret_cast<decltype(g_api.field)>(dlsym(h, name)); \
  if (!g_api.field) {                                                  \
    g_why = "missing NCCL symbol " name;                               \
    return;                                                            \
  }
  OOO_SYM(GetUniqueId, "ncclGetUniqueId")
  OOO_SYM(CommInitRank, "ncclCommInitRank")
  OOO_SYM(AllReduce, "ncclAllReduce")
  OOO_SYM(Send, "ncclSend")
  OOO_SYM(Recv, "ncclRecv")
  OOO_SYM(GroupStart, "ncclGroupStart")
  OOO_SYM(GroupEnd, "ncclGroupEnd")
  OOO_SYM(CommDestroy, "ncclCommDestroy")
  OOO_SYM(CommAbort, "ncclCommAbort")
  OOO_SYM(CommGetAsyncError, "ncclCommGetAsyncError")
  OOO_SYM(GetErrorString, "ncclGetErrorString")
  OOO_SYM(GetVersion, "ncclGetVersion")
#undef OOO_SYM
  g_api.CommInitRankConfig =
      reinterpret_cast<decltype(g_api.CommInitRankConfig)>(dlsym(h, "ncclCommInitRankConfig"));
  g_api.ok = true;
  g_why = "";
}
}  // namespace

const NcclApi *nccl_api(const char **why) {
  std::call_once(g_once, load);
  if (why) *why = g_why;
  return g_api.ok ? &g_api : nullptr;
}

}  // namespace ooo
