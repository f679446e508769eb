#include <cstdio>
__global__ void k() {
  unsigned m = 0b1011010u; // bits 1,3,4,6
  if (threadIdx.x == 0) {
    for (int base = 0; base < 8; ++base)
      for (int off = -2; off <= 3; ++off)
        printf("fns(m=0x%x, base=%d, off=%d) = %d\n", m, base, off, (int)__fns(m, base, off));
  }
}
int main() { k<<<1,32>>>(); cudaDeviceSynchronize(); return 0; }
