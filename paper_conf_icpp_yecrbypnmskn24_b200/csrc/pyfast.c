/* pyfast.c -- CPython fast path for the per-update calls of the binding
 * (viper_publish / viper_acquire_latest / viper_release).  Argument marshalling
 * only, like the ctypes binding: it resolves the same libviper.so symbols with
 * dlsym and forwards plain integers, saving the ~1.3 us per direction that
 * ctypes argument conversion costs on the C1 update (~20 us). */
#define PY_SSIZE_T_CLEAN
#include <Python.h>
#include <dlfcn.h>
#include <stdint.h>

typedef int32_t viper_status;
typedef struct {
    uint64_t version;
    int32_t slot;
    int32_t ntensors;
    void *const *dev_ptrs;
    uint64_t ticket;
} viper_view;

static viper_status (*p_publish)(void *, uint64_t, void *);
static viper_status (*p_acquire)(void *, uint64_t, int64_t, viper_view *);
static viper_status (*p_release)(void *, const viper_view *, void *);

static PyObject *fast_init(PyObject *self, PyObject *args) {
    const char *path;
    if (!PyArg_ParseTuple(args, "s", &path)) return NULL;
    void *h = dlopen(path, RTLD_NOW | RTLD_GLOBAL);
    if (!h) return PyErr_Format(PyExc_ImportError, "dlopen(%s): %s", path, dlerror());
    p_publish = dlsym(h, "viper_publish");
    p_acquire = dlsym(h, "viper_acquire_latest");
    p_release = dlsym(h, "viper_release");
    if (!p_publish || !p_acquire || !p_release) return PyErr_Format(PyExc_ImportError, "missing viper symbols");
    Py_RETURN_NONE;
}

static PyObject *fast_publish(PyObject *self, PyObject *const *args, Py_ssize_t n) {
    if (n != 3) return PyErr_Format(PyExc_TypeError, "publish(handle, version, stream)");
    void *h = PyLong_AsVoidPtr(args[0]);
    const uint64_t v = PyLong_AsUnsignedLongLong(args[1]);
    void *st = args[2] == Py_None ? NULL : PyLong_AsVoidPtr(args[2]);
    if (PyErr_Occurred()) return NULL;
    viper_status r;
    Py_BEGIN_ALLOW_THREADS r = p_publish(h, v, st);
    Py_END_ALLOW_THREADS return PyLong_FromLong(r);
}

static PyObject *fast_acquire(PyObject *self, PyObject *const *args, Py_ssize_t n) {
    if (n != 3) return PyErr_Format(PyExc_TypeError, "acquire(handle, min_version, timeout_us)");
    void *h = PyLong_AsVoidPtr(args[0]);
    const uint64_t mv = PyLong_AsUnsignedLongLong(args[1]);
    const int64_t to = PyLong_AsLongLong(args[2]);
    if (PyErr_Occurred()) return NULL;
    viper_view v = {0, 0, 0, NULL, 0};
    viper_status r;
    Py_BEGIN_ALLOW_THREADS r = p_acquire(h, mv, to, &v);
    Py_END_ALLOW_THREADS return Py_BuildValue("iKiiKK", r, (unsigned long long)v.version, v.slot, v.ntensors,
                                              (unsigned long long)(uintptr_t)v.dev_ptrs,
                                              (unsigned long long)v.ticket);
}

static PyObject *fast_release(PyObject *self, PyObject *const *args, Py_ssize_t n) {
    if (n != 7) return PyErr_Format(PyExc_TypeError, "release(handle, version, slot, ntensors, ptrs, ticket, stream)");
    void *h = PyLong_AsVoidPtr(args[0]);
    viper_view v;
    v.version = PyLong_AsUnsignedLongLong(args[1]);
    v.slot = (int32_t)PyLong_AsLong(args[2]);
    v.ntensors = (int32_t)PyLong_AsLong(args[3]);
    v.dev_ptrs = (void *const *)PyLong_AsVoidPtr(args[4]);
    v.ticket = PyLong_AsUnsignedLongLong(args[5]);
    void *st = args[6] == Py_None ? NULL : PyLong_AsVoidPtr(args[6]);
    if (PyErr_Occurred()) return NULL;
    viper_status r;
    Py_BEGIN_ALLOW_THREADS r = p_release(h, &v, st);
    Py_END_ALLOW_THREADS return PyLong_FromLong(r);
}

static PyMethodDef methods[] = {
    {"init", fast_init, METH_VARARGS, "resolve libviper.so symbols"},
    {"publish", (PyCFunction)(void (*)(void))fast_publish, METH_FASTCALL, "viper_publish"},
    {"acquire", (PyCFunction)(void (*)(void))fast_acquire, METH_FASTCALL, "viper_acquire_latest"},
    {"release", (PyCFunction)(void (*)(void))fast_release, METH_FASTCALL, "viper_release"},
    {NULL, NULL, 0, NULL}};

static struct PyModuleDef mod = {PyModuleDef_HEAD_INIT, "_fast", "libviper.so fast-call shim", -1, methods};

PyMODINIT_FUNC PyInit__fast(void) { return PyModule_Create(&mod); }
