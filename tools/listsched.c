/* List-scheduling makespan for tools/fit_model.py: CTAs (entry i repeated
 * mult times, in launch order) are dispatched onto `slots` identical slots,
 * each to the earliest-free slot (the block scheduler's behaviour). */
#include <stdlib.h>
double makespan(int n, const double* t, int mult, int slots, double* heap) {
    int sz = slots;
    for (int i = 0; i < sz; ++i) heap[i] = 0.0;
    for (int i = 0; i < n; ++i)
        for (int m = 0; m < mult; ++m) {
            /* pop min (root), push root + t[i]: replace root and sift down */
            double v = heap[0] + t[i];
            int k = 0;
            for (;;) {
                int l = 2 * k + 1, r = l + 1, s = k;
                double sv = v;
                if (l < sz && heap[l] < sv) { s = l; sv = heap[l]; }
                if (r < sz && heap[r] < sv) { s = r; sv = heap[r]; }
                if (s == k) break;
                heap[k] = heap[s];
                k = s;
            }
            heap[k] = v;
        }
    double mx = 0;
    for (int i = 0; i < sz; ++i) if (heap[i] > mx) mx = heap[i];
    return mx;
}
