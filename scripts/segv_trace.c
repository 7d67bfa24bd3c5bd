#include <execinfo.h>
#include <signal.h>
#include <stdio.h>
#include <stdlib.h>
#include <unistd.h>
static void h(int sig) {
  void *b[64];
  int n = backtrace(b, 64);
  fprintf(stderr, "[segv_trace] signal %d, native backtrace:\n", sig);
  backtrace_symbols_fd(b, n, 2);
  _exit(128 + sig);
}
__attribute__((constructor)) static void init(void) { signal(SIGSEGV, h); signal(SIGBUS, h); }
